// api.cu -- the C-ABI (include/sieve.h) and the host orchestrator of the stratification path.
//
// The orchestrator sequences the device passes and takes the few replicated, exact host
// decisions the paper's method needs between them:
//   pass A moments -> [AR-1] -> tiers (exact u256 CoV test) -> Tier-3 compaction ->
//   radix sort -> prefix sums -> rounds { bandwidth h (host fp64, Scott [36]) -> KDE ->
//   [AR-2] -> valleys -> part moments -> [AR-3] -> exact CoV test per part } ->
//   stratum table (kernel, lo) -> pass B assignment + (stratum, CTA) statistics -> [AR-4] ->
//   representatives -> representatives' (x, y) -> [AR-5].
// Every [AR-*] is an exact u64-lane all-reduce (limbs for u128), so each rank takes identical
// decisions and the strata are byte-identical for any number of ranks.
#include <math.h>
#include <stdio.h>
#include <string.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <string>
#include <vector>

#include "comm.h"
#include "kernels.cuh"

// ------------------------------------------------------------------------------------------
// errors
// ------------------------------------------------------------------------------------------
static thread_local std::string t_err;
void sv_set_error(const std::string& msg) { t_err = msg; }
int sv_fail(int code, const std::string& msg) { t_err = msg; return code; }
int sv_cuda(cudaError_t e, const char* what, int line) {
  char buf[512];
  snprintf(buf, sizeof buf, "CUDA error %s (%s) at api line %d: %s", cudaGetErrorName(e),
           cudaGetErrorString(e), line, what);
  t_err = buf;
  return e == cudaErrorMemoryAllocation ? SIEVE_ENOMEM : SIEVE_ECUDA;
}
extern "C" const char* sieve_last_error(void) { return t_err.c_str(); }
extern "C" const char* sieve_version(void) { return "sieve-b200 0.1 (sm_100a)"; }

cudaError_t sv_set_smem(const void* fn, int bytes) {
  // small lock-free cache of (kernel, device) -> largest size already set; a race only repeats
  // an idempotent driver call
  struct E { std::atomic<const void*> fn; std::atomic<int> dev, bytes; };
  static E cache[64];
  int dev = 0;
  cudaGetDevice(&dev);
  for (auto& e : cache) {
    const void* f = e.fn.load(std::memory_order_acquire);
    if (f == fn && e.dev.load() == dev) {
      if (e.bytes.load() >= bytes) return cudaSuccess;
      cudaError_t r = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
      if (r == cudaSuccess) e.bytes.store(bytes);
      return r;
    }
    if (f == nullptr) {
      cudaError_t r = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
      const void* expect = nullptr;
      if (r == cudaSuccess && e.fn.compare_exchange_strong(expect, fn)) { e.dev.store(dev); e.bytes.store(bytes); }
      return r;
    }
  }
  return cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
}

int sv_num_sms() {
  static int cache[64] = {0};
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= 64) dev = 0;
  if (!cache[dev]) {
    int v = 0;
    cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev);
    cache[dev] = v > 0 ? v : 148;
  }
  return cache[dev];
}

extern "C" void sieve_u128_to_limbs(uint64_t lo, uint64_t hi, uint64_t limbs[4]) {
  limbs_from_u128(lo, hi, (u64*)limbs);
}
extern "C" void sieve_limbs_to_u128(const uint64_t limbs[4], uint64_t* lo, uint64_t* hi) {
  limbs_to_u128((const u64*)limbs, (u64*)lo, (u64*)hi);
}

// ------------------------------------------------------------------------------------------
// handles
// ------------------------------------------------------------------------------------------
#define CTX_MAGIC 0x51E7C7A0u
#define TRACE_MAGIC 0x51E7C7A1u
#define STRATA_MAGIC 0x51E7C7A2u

struct PhaseAcc { double ms = 0; u64 calls = 0; u64 work = 0; };
struct PendingEv { int ph; cudaEvent_t a, b; };

// the allocator a device buffer came from: it is always released through the same one, even
// after sieve_ctx_set_allocator changed the context's hooks
struct Owner {
  sieve_free_fn ff = nullptr;  // nullptr: cudaMallocAsync / cudaFreeAsync
  void* user = nullptr;
};
// a read-back staged in pinned memory: copied into its host destination at the next sync
struct CtxPend { void* dst; void* pinned; size_t bytes; };

struct sieve_ctx_s {
  uint32_t magic = CTX_MAGIC;
  int device = 0;
  cudaStream_t stream = 0;
  int rank = 0, world = 1;
  Comm* comm = nullptr;
  sieve_alloc_fn af = nullptr;
  sieve_free_fn ff = nullptr;
  void* user = nullptr;
  bool timing = false;
  PhaseAcc acc[SIEVE_PHASE_COUNT];
  std::vector<PendingEv> pending;
  std::vector<cudaEvent_t> ev_pool;
  // per-call scratch arena: every temporary of a stratify / predict call is bump-allocated
  // from one device buffer that is reset at the start of the next call (all work of a call is
  // ordered on the ctx stream and synchronised before it returns).  A call that overflows
  // gets the overflow from the allocator and the arena grows to the high-water mark, so
  // steady-state calls never touch the allocator (no pool remapping, no fragmentation).
  char* arena = nullptr;
  Owner arena_owner;
  size_t arena_cap = 0, arena_off = 0, arena_hw = 0;
  std::vector<std::pair<void*, Owner>> overflow;
  // the same scheme in pinned host memory for the orchestrator's staged copies
  char* pin = nullptr;
  size_t pin_cap = 0, pin_off = 0, pin_hw = 0;
  std::vector<void*> pin_overflow;
  std::vector<CtxPend> pend;
  cudaEvent_t ev_moments = nullptr;   // pass A's deferred read-back
  // SIEVE_HOST_TIMING: host-side accounting of the synchronisations of a call
  int hs_n = 0;
  bool count_terms = true;  // in-window KDE term count (sieve_ctx_set_term_count)
  // mapped (zero-copy) pinned host memory: kernels write each round's part results here, in two
  // buffers used alternately, so one batch's records stay readable while the next batch runs
  u64* mapped[2] = {nullptr, nullptr};
  size_t mapped_cap[2] = {0, 0};
  u64* scan_state = nullptr;   // single-pass scans (sort.cu), zero-initialised at creation
  double hs_wait = 0, hs_between = 0;
  std::string hs_list;
  std::chrono::steady_clock::time_point hs_last{};
};

static std::atomic<unsigned long long> g_launches{0};
void sv_count_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }
extern "C" uint64_t sieve_kernel_launches(void) { return g_launches.load(); }

// CUDA events around a phase on the ctx stream (only when timing is enabled)
struct PhaseTimer {
  sieve_ctx_s* c;
  int ph;
  cudaEvent_t a = nullptr;
  PhaseTimer(sieve_ctx_s* cc, int p, u64 work) : c(cc), ph(p) {
    if (!c->timing) return;
    a = take();
    cudaEventRecord(a, c->stream);
    c->acc[ph].calls++;
    c->acc[ph].work += work;
  }
  cudaEvent_t take() {
    if (c->ev_pool.empty()) { cudaEvent_t e; cudaEventCreate(&e); return e; }
    cudaEvent_t e = c->ev_pool.back();
    c->ev_pool.pop_back();
    return e;
  }
  void stop() {
    if (!a) return;
    cudaEvent_t b = take();
    cudaEventRecord(b, c->stream);
    c->pending.push_back({ph, a, b});
    a = nullptr;
  }
  ~PhaseTimer() { stop(); }
};

// after the stream is synchronised: fold the recorded event pairs into the accumulators
static void resolve_timing(sieve_ctx_s* c) {
  for (auto& p : c->pending) {
    float ms = 0;
    if (cudaEventElapsedTime(&ms, p.a, p.b) == cudaSuccess) c->acc[p.ph].ms += ms;
    c->ev_pool.push_back(p.a);
    c->ev_pool.push_back(p.b);
  }
  c->pending.clear();
}

extern "C" int sieve_ctx_set_timing(sieve_ctx ctx, int enable) {
  if (!ctx || ctx->magic != CTX_MAGIC) return sv_fail(SIEVE_EINVAL, "bad ctx");
  ctx->timing = enable != 0;
  for (auto& a : ctx->acc) a = PhaseAcc();
  return SIEVE_OK;
}

extern "C" int sieve_ctx_set_term_count(sieve_ctx ctx, int enable) {
  if (!ctx || ctx->magic != CTX_MAGIC) return sv_fail(SIEVE_EINVAL, "bad ctx");
  ctx->count_terms = enable != 0;
  return SIEVE_OK;
}

extern "C" int sieve_timing_get(sieve_ctx ctx, uint32_t phase, double* ms, uint64_t* calls, uint64_t* work) {
  if (!ctx || ctx->magic != CTX_MAGIC || phase >= SIEVE_PHASE_COUNT) return sv_fail(SIEVE_EINVAL, "bad ctx or phase");
  if (ms) *ms = ctx->acc[phase].ms;
  if (calls) *calls = ctx->acc[phase].calls;
  if (work) *work = ctx->acc[phase].work;
  return SIEVE_OK;
}

static std::atomic<u64> g_trace_serial{0};
struct sieve_trace_s {
  uint32_t magic = TRACE_MAGIC;
  u64 serial = ++g_trace_serial;   // unique per trace handle (a freed handle's address may recur)
  sieve_ctx ctx = nullptr;
  u64 n = 0, first_id = 0;
  u32 K = 0;
  u32* kid = nullptr;
  u64* x = nullptr;
  u32* cta = nullptr;
  u64* y = nullptr;
  bool owned = true;
  Owner owner;                     // allocator of the owned columns
  std::vector<std::string> names;  // kernel names by id (traces loaded from CSV)
};

struct SegDebug {
  sieve_segment meta;
  std::vector<u64> dlo, dhi, cuts;
};

struct sieve_strata_s {
  uint32_t magic = STRATA_MAGIC;
  sieve_ctx ctx = nullptr;
  std::vector<sieve_stratum> st;
  std::vector<SegDebug> segs;
  bool keep_debug = false;
  u32 G = 0;
  u32 rounds = 0;
  u64 kde_terms = 0, kde_evaluated = 0;
  u128 total_instr = 0, c_meas = 0;
  bool has_cycles = false;
  // the prediction from the trace's own cycles, computed with the representatives (same kernel,
  // same inputs as sieve_predict would use); valid for the trace it was stratified from
  bool pred_ok = false;
  u64 pred_serial = 0;
  double pred_r[4] = {0, 0, 0, 0};
};

static bool ctx_ok(sieve_ctx c) { return c && c->magic == CTX_MAGIC; }
// a stratum-table buffer kept per thread between results (a result's table is ~100 B per stratum)
static std::vector<sieve_stratum>& spare_strata() {
  static thread_local std::vector<sieve_stratum> v;
  return v;
}
static bool trace_ok(sieve_trace t) { return t && t->magic == TRACE_MAGIC && ctx_ok(t->ctx); }
static bool strata_ok(sieve_strata s) { return s && s->magic == STRATA_MAGIC; }

// device memory through the ctx allocator (default: stream-ordered cudaMallocAsync)
static int dalloc(sieve_ctx c, void** p, size_t bytes) {
  *p = nullptr;
  if (bytes == 0) bytes = 16;
  if (c->af) {
    *p = c->af(bytes, (void*)c->stream, c->user);
    if (!*p) return sv_fail(SIEVE_ENOMEM, "allocator hook returned NULL");
    return SIEVE_OK;
  }
  SV_CUDA(cudaMallocAsync(p, bytes, c->stream));
  return SIEVE_OK;
}
static Owner cur_owner(sieve_ctx c) { return Owner{c->ff, c->user}; }
static void dfree(sieve_ctx c, const Owner& o, void* p) {
  if (!p) return;
  if (o.ff) o.ff(p, (void*)c->stream, o.user);
  else cudaFreeAsync(p, c->stream);
}

static int pin_alloc(sieve_ctx c, void** p, size_t bytes) {
  bytes = (bytes + 255) / 256 * 256;
  if (bytes == 0) bytes = 256;
  size_t off = c->pin_off;
  c->pin_off += bytes;
  if (c->pin_off > c->pin_hw) c->pin_hw = c->pin_off;
  if (c->pin_off <= c->pin_cap) { *p = c->pin + off; return SIEVE_OK; }
  SV_CUDA(cudaHostAlloc(p, bytes, cudaHostAllocDefault));
  c->pin_overflow.push_back(*p);
  return SIEVE_OK;
}

// a mapped pinned host buffer of at least `bytes` (grown, never shrunk; its contents are only
// valid between a kernel that writes it and the host's read after the next stream sync)
static int mapped_get(sieve_ctx c, int slot, size_t bytes, u64** host, u64** dev) {
  if (bytes > c->mapped_cap[slot]) {
    SV_CUDA(cudaStreamSynchronize(c->stream));  // the old buffer may still be written
    if (c->mapped[slot]) cudaFreeHost(c->mapped[slot]);
    c->mapped[slot] = nullptr;
    c->mapped_cap[slot] = 0;
    size_t want = bytes + bytes / 2 + 4096;
    void* p;
    SV_CUDA(cudaHostAlloc(&p, want, cudaHostAllocMapped | cudaHostAllocPortable));
    c->mapped[slot] = (u64*)p;
    c->mapped_cap[slot] = want;
  }
  void* d;
  SV_CUDA(cudaHostGetDevicePointer(&d, c->mapped[slot], 0));
  *host = c->mapped[slot];
  *dev = (u64*)d;
  return SIEVE_OK;
}

static int arena_reset(sieve_ctx c) {
  // pinned staging: every copy of the previous call completed before it returned
  c->pend.clear();
  for (void* p : c->pin_overflow) cudaFreeHost(p);
  c->pin_overflow.clear();
  if (c->pin_hw > c->pin_cap) {
    if (c->pin) cudaFreeHost(c->pin);
    c->pin = nullptr;
    c->pin_cap = 0;
    size_t want = c->pin_hw + c->pin_hw / 4 + 4096;
    void* p;
    SV_CUDA(cudaHostAlloc(&p, want, cudaHostAllocDefault));
    c->pin = (char*)p;
    c->pin_cap = want;
  }
  c->pin_off = 0;
  c->pin_hw = 0;
  for (auto& q : c->overflow) dfree(c, q.second, q.first);
  c->overflow.clear();
  if (c->arena_hw > c->arena_cap) {
    if (c->arena) dfree(c, c->arena_owner, c->arena);
    c->arena = nullptr;
    c->arena_cap = 0;
    size_t want = c->arena_hw + c->arena_hw / 8;
    void* p;
    SV_TRY(dalloc(c, &p, want));
    c->arena = (char*)p;
    c->arena_owner = cur_owner(c);
    c->arena_cap = want;
  }
  c->arena_off = 0;
  c->arena_hw = 0;
  return SIEVE_OK;
}

static int arena_alloc(sieve_ctx c, void** p, size_t bytes) {
  bytes = (bytes + 255) / 256 * 256;
  if (bytes == 0) bytes = 256;
  size_t off = c->arena_off;
  c->arena_off += bytes;
  if (c->arena_off > c->arena_hw) c->arena_hw = c->arena_off;
  if (c->arena_off <= c->arena_cap) { *p = c->arena + off; return SIEVE_OK; }
  SV_TRY(dalloc(c, p, bytes));  // overflow this call; the arena grows at the next reset
  c->overflow.push_back({*p, cur_owner(c)});
  return SIEVE_OK;
}

// a temporary device array of one call (freed wholesale at the next call's arena reset)
template <typename T>
struct DBuf {
  sieve_ctx c = nullptr;
  T* p = nullptr;
  size_t n = 0;
  DBuf() {}
  explicit DBuf(sieve_ctx cc) : c(cc) {}
  DBuf(const DBuf&) = delete;
  DBuf& operator=(const DBuf&) = delete;
  void release() { p = nullptr; n = 0; }
  int alloc(size_t count) {
    n = count;
    void* q;
    int st = arena_alloc(c, &q, count * sizeof(T));
    p = (T*)q;
    return st;
  }
  T* get() const { return p; }
};

// ------------------------------------------------------------------------------------------
// contexts
// ------------------------------------------------------------------------------------------
extern "C" int sieve_get_unique_id(uint8_t out[128]) {
  if (!out) return sv_fail(SIEVE_EINVAL, "out is NULL");
  return nccl_unique_id(out);
}

static int ctx_common(int dev, void* stream, sieve_ctx* out, sieve_ctx_s** c) {
  if (!out) return sv_fail(SIEVE_EINVAL, "out is NULL");
  *out = nullptr;
  int ndev = 0;
  SV_CUDA(cudaGetDeviceCount(&ndev));
  if (dev < 0 || dev >= ndev) return sv_fail(SIEVE_EINVAL, "bad cuda_device");
  SV_CUDA(cudaSetDevice(dev));
  // keep freed pool memory for the next call (repeated stratify calls do not re-map)
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
    uint64_t thr = UINT64_MAX;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
  }
  *c = new sieve_ctx_s();
  (*c)->device = dev;
  (*c)->stream = (cudaStream_t)stream;
  void* st = nullptr;
  const size_t sb = (SCAN_SP_MAX_TILES + 2) * sizeof(u64);
  cudaError_t e = cudaMalloc(&st, sb);
  if (e == cudaSuccess) e = cudaMemset(st, 0, sb);
  if (e != cudaSuccess) { if (st) cudaFree(st); delete *c; return sv_cuda(e, "scan state", __LINE__); }
  (*c)->scan_state = (u64*)st;
  return SIEVE_OK;
}

extern "C" int sieve_ctx_create(int cuda_device, void* cuda_stream, int rank, int world,
                                const uint8_t* nccl_id, sieve_ctx* out) {
  if (world < 1 || rank < 0 || rank >= world) return sv_fail(SIEVE_EINVAL, "bad rank/world");
  if (world > 1 && nccl_id == nullptr) return sv_fail(SIEVE_EINVAL, "world > 1 needs an nccl_id");
  sieve_ctx_s* c;
  SV_TRY(ctx_common(cuda_device, cuda_stream, out, &c));
  c->rank = rank;
  c->world = world;
  if (nccl_id) {  // world == 1 with an id: a one-rank NCCL communicator (exercises the NCCL path)
    int st = nccl_comm_create(rank, world, nccl_id, &c->comm);
    if (st != SIEVE_OK) { delete c; return st; }
  }
  *out = c;
  return SIEVE_OK;
}

extern "C" int sieve_ctx_create_in_group(int cuda_device, void* cuda_stream, sieve_group g, int rank,
                                         sieve_ctx* out) {
  sieve_ctx_s* c;
  SV_TRY(ctx_common(cuda_device, cuda_stream, out, &c));
  int st = group_comm_create(g, rank, &c->comm);
  if (st != SIEVE_OK) { delete c; return st; }
  c->rank = c->comm->rank;
  c->world = c->comm->world;
  *out = c;
  return SIEVE_OK;
}

extern "C" int sieve_ctx_set_allocator(sieve_ctx ctx, sieve_alloc_fn a, sieve_free_fn f, void* user) {
  if (!ctx_ok(ctx) || (!a) != (!f)) return sv_fail(SIEVE_EINVAL, "bad ctx or allocator pair");
  SV_CUDA(cudaSetDevice(ctx->device));
  // the scratch arena goes back to the allocator it came from now (no call is in flight: every
  // call synchronises before it returns), so the next call grows a new one from the new hooks;
  // traces keep their owner and are released through it by sieve_trace_free
  SV_CUDA(cudaStreamSynchronize(ctx->stream));
  for (auto& q : ctx->overflow) dfree(ctx, q.second, q.first);
  ctx->overflow.clear();
  if (ctx->arena) dfree(ctx, ctx->arena_owner, ctx->arena);
  ctx->arena = nullptr;
  ctx->arena_cap = ctx->arena_off = 0;
  SV_CUDA(cudaStreamSynchronize(ctx->stream));
  ctx->af = a; ctx->ff = f; ctx->user = user;
  return SIEVE_OK;
}

extern "C" void sieve_ctx_destroy(sieve_ctx ctx) {
  if (!ctx_ok(ctx)) return;
  cudaSetDevice(ctx->device);
  for (auto& p : ctx->pending) { cudaEventDestroy(p.a); cudaEventDestroy(p.b); }
  for (auto e : ctx->ev_pool) cudaEventDestroy(e);
  for (auto& q : ctx->overflow) dfree(ctx, q.second, q.first);
  if (ctx->arena) dfree(ctx, ctx->arena_owner, ctx->arena);
  cudaStreamSynchronize(ctx->stream);
  for (void* p : ctx->pin_overflow) cudaFreeHost(p);
  if (ctx->pin) cudaFreeHost(ctx->pin);
  for (u64* m : ctx->mapped)
    if (m) cudaFreeHost(m);
  if (ctx->scan_state) cudaFree(ctx->scan_state);
  if (ctx->ev_moments) cudaEventDestroy(ctx->ev_moments);
  delete ctx->comm;
  ctx->magic = 0;
  delete ctx;
}

extern "C" void sieve_params_default(sieve_params* p) {
  if (!p) return;
  p->theta_num = 2;
  p->theta_den = 5;
  p->grid_points = 1024;
  p->valley_shift = 10;
  p->max_rounds = 64;
  p->keep_debug = 0;
  p->bw_scale = 1.06;
}

// ------------------------------------------------------------------------------------------
// trace
// ------------------------------------------------------------------------------------------
extern "C" int sieve_load_trace(sieve_ctx ctx, uint64_t n_local, uint64_t first_id, uint32_t K,
                                const uint32_t* kernel_id, const uint64_t* instr, const uint32_t* cta,
                                const uint64_t* cycles, uint32_t mem, sieve_trace* out) {
  if (!out) return sv_fail(SIEVE_EINVAL, "out is NULL");
  *out = nullptr;
  if (!ctx_ok(ctx)) return sv_fail(SIEVE_EINVAL, "bad ctx");
  if (K == 0 || K > SIEVE_MAX_K) return sv_fail(SIEVE_ERANGE, "num_kernels must be in [1, 65536]");
  if (n_local >= (1ull << 32)) return sv_fail(SIEVE_ERANGE, "n_local must be < 2^32");
  if (n_local && (!kernel_id || !instr)) return sv_fail(SIEVE_EINVAL, "kernel_id and instr are required");
  if (mem & ~15u) return sv_fail(SIEVE_EINVAL, "bad mem flags");
  bool dev = mem & SIEVE_MEM_DEVICE, adopt = mem & SIEVE_ADOPT;
  const bool kid16 = mem & SIEVE_KID16, cta16 = mem & SIEVE_CTA16;
  if (adopt && !dev) return sv_fail(SIEVE_EINVAL, "SIEVE_ADOPT needs SIEVE_MEM_DEVICE");
  if (adopt && (kid16 || cta16)) return sv_fail(SIEVE_EINVAL, "16-bit columns cannot be adopted");
  SV_CUDA(cudaSetDevice(ctx->device));
  sieve_trace_s* t = new sieve_trace_s();
  t->ctx = ctx; t->n = n_local; t->first_id = first_id; t->K = K; t->owned = !adopt;
  t->owner = cur_owner(ctx);
  if (adopt) {
    t->kid = (u32*)kernel_id; t->x = (u64*)instr; t->cta = (u32*)cta; t->y = (u64*)cycles;
  } else {
    cudaMemcpyKind kind = dev ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
    auto cp = [&](void** dst, const void* src, size_t bytes) -> int {
      if (!src) { *dst = nullptr; return SIEVE_OK; }
      SV_TRY(dalloc(ctx, dst, bytes));
      if (bytes) SV_CUDA(cudaMemcpyAsync(*dst, src, bytes, kind, ctx->stream));
      return SIEVE_OK;
    };
    // A 16-bit column is copied as it is into a temporary and widened into the u32 column after
    // ALL the copies are queued: the copy engine streams the columns back to back (a widening
    // kernel between two copies would wait for free SMs -- behind another context's KDE, say --
    // with the engine idle).  The call returns once the caller's arrays have been read (an event
    // after the last copy); the widening completes in stream order before any later work.
    struct Widen { void* tmp; u32* dst; };
    Widen wd[2];
    int nwd = 0;
    auto cp16 = [&](void** dst, const void* src) -> int {
      if (!src) { *dst = nullptr; return SIEVE_OK; }
      SV_TRY(dalloc(ctx, dst, n_local * 4));
      if (!n_local) return SIEVE_OK;
      void* tmp = nullptr;
      SV_TRY(dalloc(ctx, &tmp, n_local * 2));
      wd[nwd++] = {tmp, (u32*)*dst};
      SV_CUDA(cudaMemcpyAsync(tmp, src, n_local * 2, kind, ctx->stream));
      return SIEVE_OK;
    };
    int st = SIEVE_OK;
    if (kid16) st = cp16((void**)&t->kid, kernel_id);
    else if (st == SIEVE_OK) st = cp((void**)&t->kid, kernel_id ? kernel_id : (const uint32_t*)&t->n, n_local * 4);
    if (st == SIEVE_OK) st = cp((void**)&t->x, instr ? instr : (const uint64_t*)&t->n, n_local * 8);
    if (st == SIEVE_OK) st = cta16 ? cp16((void**)&t->cta, cta) : cp((void**)&t->cta, cta, n_local * 4);
    if (st == SIEVE_OK) st = cp((void**)&t->y, cycles, n_local * 8);
    cudaEvent_t copied = nullptr;
    if (st == SIEVE_OK && !dev) {
      cudaError_t e = cudaEventCreateWithFlags(&copied, cudaEventDisableTiming);
      if (e == cudaSuccess) e = cudaEventRecord(copied, ctx->stream);
      if (e != cudaSuccess) st = sv_cuda(e, "load event", __LINE__);
    }
    for (int i = 0; i < nwd; i++) {
      if (st == SIEVE_OK) {
        launch_widen_u16(wd[i].tmp, n_local, wd[i].dst, ctx->stream);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) st = sv_cuda(e, "16-bit column", __LINE__);
      }
      dfree(ctx, t->owner, wd[i].tmp);
    }
    if (st == SIEVE_OK) {
      cudaError_t e = copied ? cudaEventSynchronize(copied) : cudaStreamSynchronize(ctx->stream);
      if (e) st = sv_cuda(e, "load sync", __LINE__);
    }
    if (copied) cudaEventDestroy(copied);
    if (st != SIEVE_OK) { t->magic = TRACE_MAGIC; sieve_trace_free(t); return st; }
  }
  *out = t;
  return SIEVE_OK;
}

extern "C" void sieve_trace_free(sieve_trace t) {
  if (!t || t->magic != TRACE_MAGIC) return;
  if (t->owned && ctx_ok(t->ctx)) {
    cudaSetDevice(t->ctx->device);
    const Owner& o = t->owner;
    dfree(t->ctx, o, t->kid); dfree(t->ctx, o, t->x); dfree(t->ctx, o, t->cta); dfree(t->ctx, o, t->y);
    cudaStreamSynchronize(t->ctx->stream);
  }
  t->magic = 0;
  delete t;
}

// ------------------------------------------------------------------------------------------
// exact host arithmetic for the replicated decisions
// ------------------------------------------------------------------------------------------
// correctly rounded conversion to double (round to nearest even)
static double w256_to_double(W256 a) {
  int top = 3;
  while (top > 0 && a.w[top] == 0) top--;
  if (top <= 1) return (double)(((u128)a.w[1] << 64) | a.w[0]);
  int lz = __builtin_clzll(a.w[top]);
  int nbits = 64 * top + 64 - lz;
  int sh = nbits - 64;                         // >= 65 here
  // extract the 64 bits [sh, sh+64) and a sticky of the bits below
  int wq = sh / 64, bq = sh % 64;
  u64 hi64 = bq ? ((a.w[wq] >> bq) | (a.w[wq + 1] << (64 - bq))) : a.w[wq];
  bool sticky = bq ? (a.w[wq] & ((1ull << bq) - 1)) != 0 : false;
  for (int i = 0; i < wq && !sticky; i++) sticky = a.w[i] != 0;
  return ldexp((double)(hi64 | (sticky ? 1ull : 0ull)), sh);
}


// Scott's normal-reference bandwidth ([36]; A8), rounded to 16 significant bits
static double scott_h(u64 n, u128 s1, u128 s2, double bw_scale) {
  W256 v = w256_sub(w256_mul(n, s2), w256_mul(s1, s1));
  double dn = (double)n;
  double var = w256_to_double(v) / (dn * dn);
  double h_raw = (bw_scale * sqrt(var)) * pow(dn, -0.2);
  int e = ilogb(h_raw) - 15;
  return ldexp(rint(ldexp(h_raw, -e)), e);
}

static inline u128 u128_of(u64 lo, u64 hi) { return ((u128)hi << 64) | lo; }
static inline u128 limbs_u128(const u64* l) { u64 lo, hi; limbs_to_u128(l, &lo, &hi); return u128_of(lo, hi); }
static inline u32 bitlen(u64 v) { return v ? 64 - __builtin_clzll(v) : 0; }

static int allreduce(sieve_ctx c, u64* buf, size_t n, ReduceOp op) {
  if (!c->comm) return SIEVE_OK;
  return c->comm->allreduce(buf, n, op, c->stream);
}
// several all-reduces as one collective step (one NCCL group = one fused launch)
static int allreduce_group(sieve_ctx c, std::initializer_list<ARReq> reqs) {
  if (!c->comm) return SIEVE_OK;
  return c->comm->allreduce_group(reqs.begin(), (int)reqs.size(), c->stream);
}

// Host <-> device copies of the orchestrator go through a per-call PINNED staging arena: a
// copy to or from pageable memory would make cudaMemcpyAsync synchronise the stream (H2D) or
// block the host until the copy ran (D2H).  d2h only queues the copy; the data lands in the
// vector at the next sync(c), so several read-backs share one synchronisation.
static int d2h_raw(sieve_ctx c, void* dst, const void* d, size_t bytes) {
  if (!bytes) return SIEVE_OK;
  void* p;
  SV_TRY(pin_alloc(c, &p, bytes));
  launch_copy(p, d, bytes, c->stream);  // SM copy into the UVA-mapped staging (no copy engine)
  c->pend.push_back({dst, p, bytes});
  return SIEVE_OK;
}
template <typename T>
static int d2h(sieve_ctx c, std::vector<T>& h, const T* d, size_t n) {
  h.resize(n);
  return d2h_raw(c, h.data(), d, n * sizeof(T));
}
template <typename T>
static int h2d(sieve_ctx c, T* d, const std::vector<T>& h) {
  if (h.empty()) return SIEVE_OK;
  void* p;
  SV_TRY(pin_alloc(c, &p, h.size() * sizeof(T)));
  memcpy(p, h.data(), h.size() * sizeof(T));
  launch_copy(d, p, h.size() * sizeof(T), c->stream);  // SM copy from the UVA-mapped staging
  return SIEVE_OK;
}
// Several host <-> device copies of the orchestrator in ONE launch: queue them with add_h2d /
// add_d2h (staged through the pinned arena like h2d / d2h), then flush() before the kernels that
// read the uploaded tables; read-backs land in their vectors at the next sync(c).
struct CopyBatch {
  sieve_ctx c;
  CopyRegions r{};
  explicit CopyBatch(sieve_ctx cc) : c(cc) { r.k = 0; }
  int add_raw(void* dst, const void* src, size_t bytes) {
    if (!bytes) return SIEVE_OK;
    if (r.k == COPY_MAX) SV_TRY(flush());
    r.dst[r.k] = dst; r.src[r.k] = src; r.bytes[r.k] = bytes; r.k++;
    return SIEVE_OK;
  }
  template <typename T>
  int add_h2d(T* d, const std::vector<T>& h) {
    if (h.empty()) return SIEVE_OK;
    void* p;
    SV_TRY(pin_alloc(c, &p, h.size() * sizeof(T)));
    memcpy(p, h.data(), h.size() * sizeof(T));
    return add_raw(d, p, h.size() * sizeof(T));
  }
  template <typename T>
  int add_d2h(std::vector<T>& h, const T* d, size_t n) {
    h.resize(n);
    if (!n) return SIEVE_OK;
    void* p;
    SV_TRY(pin_alloc(c, &p, n * sizeof(T)));
    c->pend.push_back({h.data(), p, n * sizeof(T)});
    return add_raw(p, d, n * sizeof(T));
  }
  int flush() {
    launch_copy_multi(r, c->stream);
    r.k = 0;
    SV_CUDA(cudaGetLastError());
    return SIEVE_OK;
  }
};

static bool host_timing() {
  static const bool on = getenv("SIEVE_HOST_TIMING") != nullptr;
  return on;
}
static int sync(sieve_ctx c) {
  if (host_timing()) {
    auto t0 = std::chrono::steady_clock::now();
    if (c->hs_n) {
      double b = std::chrono::duration<double, std::milli>(t0 - c->hs_last).count();
      c->hs_between += b;
      char tmp[32];
      snprintf(tmp, sizeof tmp, " %.3f", b);
      c->hs_list += tmp;
    }
    cudaError_t e = cudaStreamSynchronize(c->stream);
    auto t1 = std::chrono::steady_clock::now();
    c->hs_wait += std::chrono::duration<double, std::milli>(t1 - t0).count();
    c->hs_n++;
    c->hs_last = t1;
    SV_CUDA(e);
  }
  SV_CUDA(cudaStreamSynchronize(c->stream));
  for (auto& q : c->pend) memcpy(q.dst, q.pinned, q.bytes);
  c->pend.clear();
  return SIEVE_OK;
}

// ------------------------------------------------------------------------------------------
// sieve_stratify
// ------------------------------------------------------------------------------------------
// an open Tier-3 segment: global value range / moments (replicated) and this rank's index
// range [b, e) in the sorted keys (local)
// rounds > 1: its values are [b, e) of `src` (sorted cell keys, x = key >> src_shift)
struct OpenSeg { u32 kid, t3rank; u64 lo, hi, n; u128 s1, s2; u64 b, e; const u64* src; u32 src_shift;
                 int node = -1; };

// The refinement tree of a theta sweep (sieve_stratify_sweep): every segment refined at the
// smallest theta of the sweep, with its parts.  Whether a part is final depends on theta only
// through its exact CoV test (lo == hi or CoV < theta), and a segment's KDE, cuts and parts
// depend only on its values, so for theta >= theta_min the strata are the frontier of this tree
// where the CoV test first holds: the refinement runs once, not once per theta.
struct SweepTree {
  struct Seg { u32 kid, round; u64 lo, hi, n; u128 s1, s2; double h; u32 p0, p1; };
  struct Part { u64 lo, hi, n; u128 s1, s2; int child; };   // child: segment index, -1 if final
  std::vector<Seg> segs;
  std::vector<Part> parts;
  std::vector<int> root;   // per kernel: its Tier-3 root segment, -1
};

// host-side wall-clock marks (SIEVE_HOST_TIMING=1 prints them to stderr): where the host
// orchestration, not the device, spends time
struct HostClock {
  bool on = host_timing();
  sieve_ctx c = nullptr;
  std::chrono::steady_clock::time_point t0 = std::chrono::steady_clock::now(), last = t0;
  std::string out;
  void mark(const char* name) {
    if (!on) return;
    auto now = std::chrono::steady_clock::now();
    char b[96];
    snprintf(b, sizeof b, " %s=%.3f", name, std::chrono::duration<double, std::milli>(now - last).count());
    out += b;
    last = now;
  }
  ~HostClock() {
    if (!on) return;
    fprintf(stderr, "[sieve host ms]%s total=%.3f syncs=%d wait=%.3f between=%.3f [%s ]\n", out.c_str(),
            std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count(),
            c ? c->hs_n : 0, c ? c->hs_wait : 0.0, c ? c->hs_between : 0.0, c ? c->hs_list.c_str() : "");
    if (c) { c->hs_n = 0; c->hs_wait = c->hs_between = 0; c->hs_list.clear(); }
  }
};
struct Fin { u32 kid, tier; u64 lo, hi, n; u128 s1; double h; u32 round; };

// the calling thread's scans use this context's single-pass scan state for the call's duration
struct ScanScope {
  explicit ScanScope(sieve_ctx c) { scan_set_state(c->scan_state); }
  ~ScanScope() { scan_set_state(nullptr); }
};

// pass A results on the host (replicated after AR-1): theta-independent, so a theta sweep or a
// tier census computes them once
struct MomentsHost {
  std::vector<u64> lanes, mm, tot, localn;
  // pass A's per-block partials on the device (arena memory of THIS call; null when cached from
  // another call or when the kernels took several shared-memory passes)
  const KMomPartial* part = nullptr;
  int part_grid = 0;
  u32 part_kt = 0;
  // device copies of the reduced moments (valid in the call that computed them)
  const u64 *d_lanes = nullptr, *d_mm = nullptr, *d_localn = nullptr;
  // deferred read-back: the host copies land after `ready` completes (moments_finish)
  cudaEvent_t ready = nullptr;
  std::vector<CtxPend> pend;
};

// ---------------- pass A: per-kernel moments + totals -------------------
static int moments_finish(sieve_ctx c, MomentsHost* M);
// Pass A.  defer = true: the read-back is queued and an event recorded, but the host does not
// wait (the caller queues more device work first and then calls moments_finish)
static int moments_pass(sieve_trace t, MomentsHost* M, bool defer = false) {
  sieve_ctx c = t->ctx;
  cudaStream_t S = c->stream;
  const u32 K = t->K;
  const u64 n = t->n;
  const u32 kt = (u32)moments_kt(K);
  const int gridA = moments_grid(kt);
  DBuf<KMomPartial> part(c);
  DBuf<u64> blk_tot(c), lanes(c), mm(c), local_n(c), tot(c);
  SV_TRY(part.alloc((size_t)gridA * kt));
  SV_TRY(blk_tot.alloc((size_t)gridA * 3));
  SV_TRY(lanes.alloc((size_t)K * MOM_LANES));
  SV_TRY(mm.alloc((size_t)K * 2));
  SV_TRY(local_n.alloc(K));
  // tot: [0..4) C_meas limbs (SUM), [4] max x (MAX), [5..8) error lanes (MAX)
  SV_TRY(tot.alloc(8));
  SV_CUDA(cudaMemsetAsync(tot.get(), 0, 8 * 8, S));
  PhaseTimer tA(c, SIEVE_PHASE_MOMENTS, n * (12 + (t->y ? 8 : 0)));
  for (u32 k0 = 0; k0 < K; k0 += kt) {
    u32 kk = std::min(kt, K - k0);
    if (n) {
      launch_moments(t->kid, t->x, t->y, n, K, k0, kk, part.get(), blk_tot.get(), tot.get() + 5,
                     gridA, S);
      launch_moments_reduce(part.get(), blk_tot.get(), gridA, k0, kk, K, lanes.get(), mm.get(),
                            local_n.get(), tot.get(), tot.get() + 4, k0 == 0, S);
    }
  }
  if (!n) {
    SV_CUDA(cudaMemsetAsync(lanes.get(), 0, (size_t)K * MOM_LANES * 8, S));
    SV_CUDA(cudaMemsetAsync(local_n.get(), 0, (size_t)K * 8, S));
    std::vector<u64> mmh(2 * (size_t)K);
    for (u32 k = 0; k < K; k++) { mmh[2 * k] = ~0ull; mmh[2 * k + 1] = 0; }
    SV_TRY(h2d(c, mm.get(), mmh));
  }
  SV_CUDA(cudaGetLastError());
  tA.stop();
  if (c->comm) {
    // AR-1, one grouped step: SUM of the limb lanes and C_meas; MAX of (min, max) per kernel with
    // the mins complemented (min(a, b) = ~max(~a, ~b)), max x and the error lanes
    launch_complement(mm.get(), K, 2, S);
    SV_TRY(allreduce_group(c, {{lanes.get(), (size_t)K * MOM_LANES, RED_SUM}, {tot.get(), 4, RED_SUM},
                               {mm.get(), (size_t)K * 2, RED_MAX}, {tot.get() + 4, 4, RED_MAX}}));
    launch_complement(mm.get(), K, 2, S);
  }
  if (K <= kt) { M->part = part.get(); M->part_grid = gridA; M->part_kt = kt; }
  M->d_lanes = lanes.get(); M->d_mm = mm.get(); M->d_localn = local_n.get();
  {
    CopyBatch cb(c);
    SV_TRY(cb.add_d2h(M->lanes, lanes.get(), (size_t)K * MOM_LANES));
    SV_TRY(cb.add_d2h(M->mm, mm.get(), (size_t)K * 2));
    SV_TRY(cb.add_d2h(M->tot, tot.get(), 8));
    SV_TRY(cb.add_d2h(M->localn, local_n.get(), K));
    SV_TRY(cb.flush());
  }
  if (defer) {
    M->pend.swap(c->pend);   // these copies complete with the event, not at the next sync(c)
    if (!c->ev_moments) SV_CUDA(cudaEventCreateWithFlags(&c->ev_moments, cudaEventDisableTiming));
    M->ready = c->ev_moments;
    SV_CUDA(cudaEventRecord(M->ready, S));
    return SIEVE_OK;
  }
  SV_TRY(sync(c));
  return moments_finish(c, M);
}

// wait for pass A's read-back (deferred: only for its event, later work keeps running) and
// check the trace's validity flags (identical on every rank: they were all-reduced)
static int moments_finish(sieve_ctx c, MomentsHost* M) {
  if (M->ready) {
    SV_CUDA(cudaEventSynchronize(M->ready));
    for (auto& q : M->pend) memcpy(q.dst, q.pinned, q.bytes);
    M->pend.clear();
    M->ready = nullptr;
  }
  if (M->tot[5]) return sv_fail(SIEVE_EINVAL, "kernel id >= num_kernels in the trace");
  if (M->tot[6]) return sv_fail(SIEVE_ERANGE, "instruction count 0 or >= 2^44 in the trace (A21)");
  return SIEVE_OK;
}

static int stratify_impl(sieve_trace t, const sieve_params* P, uint32_t* sid_out, sieve_strata_s* R,
                         const MomentsHost* cached, SweepTree* rec = nullptr,
                         const SweepTree* use = nullptr) {
  sieve_ctx c = t->ctx;
  cudaStream_t S = c->stream;
  const auto t_entry = std::chrono::steady_clock::now();
  SV_TRY(arena_reset(c));
  ScanScope scan_scope(c);
  HostClock hc;
  hc.c = c;
  if (hc.on) {
    char b[64];
    snprintf(b, sizeof b, " reset=%.3f",
             std::chrono::duration<double, std::milli>(hc.t0 - t_entry).count());
    hc.out += b;
  }
  const u32 K = t->K, G = P->grid_points;
  const u64 n = t->n;
  MomentsHost own;
  // grouped path (G <= GROUP_MAXG): the Tier-3 rows' x grouped by segment (t3rank) at the bases
  // the local counts give; radix path: tagged keys (t3rank << bx) + x in row order
  const bool grouped = G <= GROUP_MAXG && !getenv("SIEVE_CELL_RADIX");
  DBuf<u64> keys(c);
  DBuf<u32> d_t3rank(c);
  bool pre = false;   // the round-1 grouping was queued right behind pass A
  if (!cached) {
    pre = grouped && n > 0 && K <= GROUP_T3_SMEM_MAX && !getenv("SIEVE_NO_DEVICE_TIERS");
    SV_TRY(moments_pass(t, &own, pre));
    if (pre) {
      // tiers decided on the device (the same exact test the host repeats below) and the
      // round-1 grouping queued behind pass A; the host waits only for pass A's read-back and
      // takes its own decisions while the grouping runs.  The output holds at most n values.
      DBuf<u32> tab(c), cur(c);
      DBuf<char> gtmp(c);
      SV_TRY(d_t3rank.alloc(K));
      SV_TRY(tab.alloc(2 * (size_t)K + 2));   // [segment bases | kernel of each segment | counts]
      SV_TRY(cur.alloc(K));
      SV_TRY(gtmp.alloc(group_t3_temp_bytes(K)));
      SV_TRY(keys.alloc(n));
      u32* counts = tab.get() + 2 * (size_t)K;
      launch_tiers(own.d_lanes, own.d_mm, own.d_localn, K, P->theta_num, P->theta_den, d_t3rank.get(),
                   tab.get(), tab.get() + K, counts, S);
      PhaseTimer tm(c, SIEVE_PHASE_COMPACT, n * 4);
      launch_group_t3(t->kid, t->x, n, K, d_t3rank.get(), K, counts, tab.get(), cur.get(), keys.get(),
                      gtmp.get(), own.part, own.part_grid, own.part_kt, tab.get() + K, S);
      tm.stop();
      SV_CUDA(cudaGetLastError());
    }
    SV_TRY(moments_finish(c, &own));
    cached = &own;
  }
  const std::vector<u64>& h_lanes = cached->lanes;
  const std::vector<u64>& h_mm = cached->mm;
  const std::vector<u64>& h_localn = cached->localn;
  R->c_meas = limbs_u128(&cached->tot[0]);
  const u64 max_x = cached->tot[4];

  hc.mark("passA");
  // ---------------- tiers ---------------------------------------------------------
  static thread_local std::vector<Fin> fin_tl;
  std::vector<Fin>& fin = fin_tl;
  fin.clear();
  std::vector<OpenSeg> open;
  std::vector<u32> t3rank(K, 0xFFFFFFFFu);
  u32 n_t3 = 0;
  u64 n3_local = 0;
  u128 I = 0;
  for (u32 k = 0; k < K; k++) {
    const u64* L = &h_lanes[(size_t)k * MOM_LANES];
    u64 nk = L[0];
    if (!nk) continue;
    u128 s1 = limbs_u128(L + 1), s2 = limbs_u128(L + 5);
    u64 lo = h_mm[2 * k], hi = h_mm[2 * k + 1];
    I += s1;
    if (lo == hi) {                                              // Tier-1 (A4)
      fin.push_back({k, 1, lo, hi, nk, s1, 0.0, 0});
    } else if (cov_lt(nk, s1, s2, P->theta_num, P->theta_den)) { // Tier-2
      fin.push_back({k, 2, lo, hi, nk, s1, 0.0, 0});
    } else if (use) {                                            // Tier-3: the sweep's tree
      if (use->root[k] < 0) return sv_fail(SIEVE_ESTATE, "internal: sweep tree lacks a kernel");
    } else {                                                     // Tier-3 -> refinement
      t3rank[k] = n_t3++;
      // the sorted keys are grouped by t3rank: this kernel's local range follows the previous
      open.push_back({k, t3rank[k], lo, hi, nk, s1, s2, n3_local, n3_local + h_localn[k], nullptr, 0});
      n3_local += h_localn[k];
      if (rec) {
        open.back().node = (int)rec->segs.size();
        rec->root[k] = open.back().node;
        rec->segs.push_back({k, 1, lo, hi, nk, s1, s2, 0.0, 0, 0});
      }
    }
  }
  R->total_instr = I;
  // the round-1 grouping queued behind pass A was counted as its kernel-id reads (4 B/row); its
  // Tier-3 rows' x reads and grouped writes (16 B each) are known now
  if (pre && c->timing) c->acc[SIEVE_PHASE_COMPACT].work += n3_local * 16;
  const u32 n12 = (u32)fin.size();   // the Tier-1/2 strata, in kernel order
  static thread_local std::vector<std::pair<u64, u32>> t3s_tl;
  std::vector<std::pair<u64, u32>>& t3s = t3s_tl;   // Tier-3 strata keys kid << 44 | lo, index in fin
  t3s.clear();
  u32 use_rounds = 0;
  if (use) {
    // the frontier of the tree at this theta: a part whose CoV test holds (or lo == hi) is a
    // stratum, any other part was re-opened at theta_min too and its children are visited
    std::vector<int> stack;
    for (u32 k = 0; k < K; k++) {
      const u64* L = &h_lanes[(size_t)k * MOM_LANES];
      if (!L[0] || h_mm[2 * k] == h_mm[2 * k + 1]) continue;
      if (cov_lt(L[0], limbs_u128(L + 1), limbs_u128(L + 5), P->theta_num, P->theta_den)) continue;
      stack.assign(1, use->root[k]);
      while (!stack.empty()) {
        const SweepTree::Seg& g = use->segs[stack.back()];
        stack.pop_back();
        use_rounds = std::max(use_rounds, g.round);
        // parts in descending order on the stack so they are visited by ascending lo
        for (u32 q = g.p1; q-- > g.p0;) {
          const SweepTree::Part& pt = use->parts[q];
          if (pt.lo == pt.hi || cov_lt(pt.n, pt.s1, pt.s2, P->theta_num, P->theta_den)) {
            t3s.push_back({((u64)k << 44) | pt.lo, (u32)fin.size()});
            fin.push_back({k, 3, pt.lo, pt.hi, pt.n, pt.s1, g.h, g.round});
          } else {
            if (pt.child < 0) return sv_fail(SIEVE_ESTATE, "internal: sweep tree part not refined");
            stack.push_back(pt.child);
          }
        }
      }
    }
    std::sort(t3s.begin(), t3s.end());
  }

  // ---------------- Tier-3 values: compaction (unless queued behind pass A) --------------------
  const u32 bx = std::max<u32>(1, bitlen(max_x));
  DBuf<unsigned long long> counter(c);
  SV_TRY(counter.alloc(4));
  if (n_t3 && n3_local && !pre) {
    SV_TRY(d_t3rank.alloc(K));
    CopyBatch cb(c);
    SV_TRY(cb.add_h2d(d_t3rank.get(), t3rank));
    SV_TRY(keys.alloc(n3_local));
    if (!grouped) {
      SV_TRY(cb.flush());
      SV_CUDA(cudaMemsetAsync(counter.get(), 0, 8, S));
    }
    PhaseTimer tm(c, SIEVE_PHASE_COMPACT, n * 12 + n3_local * 8);
    if (grouped) {
      std::vector<u32> sb(2 * (size_t)n_t3);   // [segment bases | kernel of each segment]
      for (u32 s = 0; s < n_t3; s++) { sb[s] = (u32)open[s].b; sb[n_t3 + s] = open[s].kid; }
      DBuf<u32> d_sb(c), cur(c);
      DBuf<char> gtmp(c);
      SV_TRY(d_sb.alloc(2 * (size_t)n_t3));
      SV_TRY(cur.alloc(n_t3));
      SV_TRY(gtmp.alloc(group_t3_temp_bytes(n_t3)));
      SV_TRY(cb.add_h2d(d_sb.get(), sb));
      SV_TRY(cb.flush());
      if (n_t3 > GROUP_T3_SMEM_MAX) SV_CUDA(cudaMemsetAsync(cur.get(), 0, (size_t)n_t3 * 4, S));  // global-cursor path
      launch_group_t3(t->kid, t->x, n, K, d_t3rank.get(), n_t3, nullptr, d_sb.get(), cur.get(), keys.get(),
                      gtmp.get(), cached == &own ? own.part : nullptr, own.part_grid, own.part_kt,
                      d_sb.get() + n_t3, S);
    } else
    launch_t3_compact(t->kid, t->x, n, d_t3rank.get(), bx, keys.get(), counter.get(), S);
    SV_CUDA(cudaGetLastError());
  }
  const u64 nkeys = (n_t3 && n3_local) ? n3_local : 0;

  hc.mark("compact");
  // ---------------- refinement rounds (A6-A15) ------------------------------------------
  // Each round sorts the open segments' values by (segment, grid cell) (bucket.cu: the segmented
  // sort the KDE windows and the part moments need), evaluates the fixed-point KDE, finds the
  // valleys and reduces the candidate parts exactly.  Round 1 reads the compacted keys (open
  // segment s = Tier-3 kernel of rank s); round r > 1 reads, for each re-opened part, its range
  // of whole cells in the sorted keys of round r-1.  The packed sort key (x << ib) | cell index
  // bounds the cells of one sort by 2^(64 - bx): a round with more open segments than that runs
  // in batches (the decisions are per segment, so batching changes no result).
  DBuf<unsigned long long> terms(c);
  SV_TRY(terms.alloc(2));
  SV_CUDA(cudaMemsetAsync(terms.get(), 0, 16, S));
  u32 round = 0;
  const u32 tstride = G / 2 + 1;
  const u32 tps = div_up(G, KDE_TJ);
  const u64 max_cells = bx >= 63 ? 0 : (1ull << (64 - bx)) - 1;  // idx <= ncell must fit
  if (!grouped && !open.empty() && max_cells < G)
    return sv_fail(SIEVE_ELIMIT, "instruction counts too wide for the cell sort key");
  for (auto& o : open) { o.src = keys.get(); o.src_shift = 0; }
  // The final parts of a batch become strata on the host after the NEXT batch's kernels are
  // queued (just before its synchronisation), so that bookkeeping overlaps device work instead of
  // delaying the next round's first launch; the batch's records stay valid in their mapped
  // buffer (the next batch writes the other one).
  struct DeferredFin { const u64* rec; u32 round; std::vector<u32> part_off, kid; std::vector<double> h; };
  std::vector<DeferredFin> dfin;
  // The Tier-3 strata are also kept sorted by (kernel, lo) as they arrive -- key kid << 44 | lo
  // (x < 2^44, K <= 2^16) with their index in fin -- so the stratum order costs one merge at
  // the end.
  auto take_finals = [&]() {
    const size_t mid = t3s.size();
    for (const DeferredFin& d : dfin)
      for (size_t s = 0; s + 1 < d.part_off.size(); s++)
        for (u32 p = d.part_off[s]; p < d.part_off[s + 1]; p++) {
          const u64* L = d.rec + 1 + (size_t)p * PART_REC;  // {lanes[9], min, max, ia, ib, final}
          if (L[0] && L[MOM_LANES + 4]) {  // non-empty, and lo == hi or CoV < theta (k_part_pack)
            t3s.push_back({((u64)d.kid[s] << 44) | L[MOM_LANES], (u32)fin.size()});
            fin.push_back({d.kid[s], 3, L[MOM_LANES], L[MOM_LANES + 1], L[0], limbs_u128(L + 1), d.h[s], d.round});
          }
        }
    dfin.clear();
    std::sort(t3s.begin() + mid, t3s.end());
    std::inplace_merge(t3s.begin(), t3s.begin() + mid, t3s.end());
  };
  u32 nbatch = 0;
  while (!open.empty()) {
    round++;
    if (round > P->max_rounds) return sv_fail(SIEVE_ELIMIT, "Tier-3 refinement exceeded max_rounds");
    static thread_local std::vector<OpenSeg> next_tl;   // capacity kept across rounds and calls
    std::vector<OpenSeg>& next = next_tl;
    next.clear();
    const u32 nopen = (u32)open.size();
    u32 batch = grouped ? nopen : (u32)std::min<u64>(nopen, std::min<u64>(max_cells / G, 0xFFFFFFFEull / G));
    if (const char* e = getenv("SIEVE_SEG_BATCH"))  // test hook: force small batches
      batch = std::max<u32>(1, std::min<u32>(batch, (u32)atoi(e)));
    // batches: runs of segments with one source array, at most `batch` segments each
    std::vector<u32> bstart;
    for (u32 s = 0; s < nopen; s++)
      if (bstart.empty() || s - bstart.back() == batch || open[s].src != open[s - 1].src) bstart.push_back(s);
    bstart.push_back(nopen);
    for (size_t bi = 0; bi + 1 < bstart.size(); bi++) {
    const u32 s0 = bstart[bi];
    const u32 nseg = bstart[bi + 1] - s0;
    const OpenSeg* op = open.data() + s0;
    const u64 ncell = (u64)nseg * G;
    const u32 ib = std::max<u32>(1, bitlen(ncell));
    hc.mark("r0");
    std::vector<SegDev> hs(nseg);
    std::vector<double> hh(nseg);
    static thread_local std::vector<BucketChunk> chunks_tl;   // capacity kept across rounds
    static thread_local std::vector<u32> seg_chunk_tl;
    std::vector<BucketChunk>& chunks = chunks_tl;
    std::vector<u32>& seg_chunk = seg_chunk_tl;   // grouped path: first chunk of every segment
    chunks.clear();
    seg_chunk.clear();
    u64 maxlen = 0;  // largest segment (local values)
    u64 nsup = 0;    // grouped path: values of the segments' source ranges
    // The bandwidths (a glibc pow each, A8) are needed first by the KDE: on the grouped path
    // without the in-window count they are computed while the cell grouping runs (the grouping
    // only reads lo, hi and the cell estimate) and uploaded with a second copy.
    const bool late_h = grouped && !c->count_terms;
    auto set_h = [&](u32 s) {
      const OpenSeg& o = op[s];
      const double h = scott_h(o.n, o.s1, o.s2, P->bw_scale);
      hh[s] = h;
      hs[s].h = h;
      hs[s].inv_h = 1.0 / h;
    };
    for (u32 s = 0; s < nseg; s++) {
      const OpenSeg& o = op[s];
      if (late_h) { hh[s] = hs[s].h = hs[s].inv_h = 0.0; } else { set_h(s); }
      hs[s].lo = o.lo;
      hs[s].hi = o.hi;
      hs[s].cq = (double)(G - 1) / (double)(o.hi - o.lo);
      hs[s].cm = cell_margin(o.lo, o.hi, G);
      u64 len = round == 1 ? h_localn[o.kid] : o.e - o.b;
      maxlen = std::max(maxlen, len);
      if (grouped) {  // every round reads each segment's contiguous source range [b, e)
        seg_chunk.push_back((u32)chunks.size());
        nsup += o.e - o.b;
        for (u64 b = o.b; b < o.e; b += GROUP_CH)
          chunks.push_back({s, (u32)std::min<u64>(GROUP_CH, o.e - b), b});
      } else if (round > 1) {
        for (u64 b = o.b; b < o.e; b += BK_CHUNK)
          chunks.push_back({s, (u32)std::min<u64>(BK_CHUNK, o.e - b), b});
      }
    }
    if (grouped) seg_chunk.push_back((u32)chunks.size());
    if (round == 1)  // the open segments are the Tier-3 kernels in t3rank order
      for (u32 s = 0; s < nseg; s++)
        if (op[s].t3rank != s0 + s) return sv_fail(SIEVE_ESTATE, "internal: round-1 segment order");
    const u64* src = op[0].src;  // one source per batch (see bstart)
    const u32 src_shift = op[0].src_shift;
    const u64 nin = grouped ? nsup : (round == 1 ? nkeys : (u64)chunks.size() * BK_CHUNK);
    const u32 vsh = grouped ? 0 : ib;  // the grouped values are raw x; cell keys carry x above ib
    DBuf<SegDev> segs(c);
    DBuf<double> gtab(c);
    DBuf<u32> off(c);
    DBuf<u64> ck(c);
    DBuf<BucketChunk> d_chunks(c);
    SV_TRY(segs.alloc(nseg));
    hc.mark("segs");
    CopyBatch rcb(c);   // this round's tables: one upload
    SV_TRY(rcb.add_h2d(segs.get(), hs));
    SV_TRY(gtab.alloc(ncell));
    SV_TRY(off.alloc(ncell + 1));
    SV_TRY(ck.alloc(std::max<u64>(nin, 1)));
    if (grouped) {
      const u32 nch = (u32)chunks.size();
      DBuf<unsigned short> cells(c);
      DBuf<u32> hist(c), rel(c), tot(c), d_sc(c);
      DBuf<char> stemp(c);
      SV_TRY(cells.alloc((size_t)std::max<u32>(nch, 1) * GROUP_CH));
      SV_TRY(hist.alloc((size_t)std::max<u32>(nch, 1) * G));
      SV_TRY(rel.alloc((size_t)std::max<u32>(nch, 1) * G));
      SV_TRY(tot.alloc(ncell));
      SV_TRY(d_sc.alloc(nseg + 1));
      SV_TRY(stemp.alloc(scan_u32_temp_bytes(ncell)));
      if (nch) {
        SV_TRY(d_chunks.alloc(nch));
        SV_TRY(rcb.add_h2d(d_chunks.get(), chunks));
      }
      SV_TRY(rcb.add_h2d(d_sc.get(), seg_chunk));
      // a segment of more than WALK_MIN_CHUNKS chunks: the per-cell walk in groups of WALK_GROUP
      // (parallel over groups; one thread per (segment, cell) would walk thousands of chunks at
      // C5: 7.5 -> 5.0 ms; C4's largest segments, 76 chunks, keep the single walk)
      u32 max_sc = 0, wgsz = WALK_GROUP, wmin = WALK_MIN_CHUNKS;
      if (const char* e = getenv("SIEVE_WALK_GROUP")) {   // test hook: smaller groups, always
        wgsz = std::max(1, atoi(e));
        wmin = wgsz;
      }
      for (u32 q = 0; q < nseg; q++) max_sc = std::max(max_sc, seg_chunk[q + 1] - seg_chunk[q]);
      DBuf<uint2> d_grp(c);
      DBuf<u32> d_sg(c), d_gs(c);
      WalkGroups wg{nullptr, nullptr, 0, nullptr};
      if (max_sc > wmin) {
        std::vector<uint2> grp;
        std::vector<u32> sg(nseg + 1);
        for (u32 q = 0; q < nseg; q++) {
          sg[q] = (u32)grp.size();
          for (u32 k = seg_chunk[q]; k < seg_chunk[q + 1]; k += wgsz)
            grp.push_back(make_uint2(k, std::min<u32>(k + wgsz, seg_chunk[q + 1])));
        }
        sg[nseg] = (u32)grp.size();
        SV_TRY(d_grp.alloc(std::max<size_t>(grp.size(), 1)));
        SV_TRY(d_sg.alloc(nseg + 1));
        SV_TRY(d_gs.alloc(std::max<size_t>(grp.size(), 1) * G));
        if (!grp.empty()) SV_TRY(rcb.add_h2d(d_grp.get(), grp));
        SV_TRY(rcb.add_h2d(d_sg.get(), sg));
        wg = WalkGroups{d_grp.get(), d_sg.get(), (u32)grp.size(), d_gs.get()};
      }
      SV_TRY(rcb.flush());
      hc.mark("up");
      PhaseTimer tm(c, SIEVE_PHASE_SORT, nin * 36 + (u64)nch * G * 16);
      launch_grid_tab(segs.get(), nseg, G, gtab.get(), S);
      launch_cell_group(d_chunks.get(), nch, src, segs.get(), nseg, G, d_sc.get(), cells.get(), hist.get(),
                        rel.get(), tot.get(), off.get(), stemp.get(), ck.get(),
                        c->count_terms ? terms.get() : nullptr, S, wg.ngrp ? &wg : nullptr);
      SV_CUDA(cudaGetLastError());
      if (late_h) {  // the bandwidths, while the grouping runs; the KDE reads them from this copy
        for (u32 s = 0; s < nseg; s++) set_h(s);
        CopyBatch hcb(c);
        SV_TRY(hcb.add_h2d(segs.get(), hs));
        SV_TRY(hcb.flush());
      }
    } else
    {
      DBuf<char> tmp(c);
      SV_TRY(tmp.alloc(radix_sort_temp_bytes(nin, false, (int)ib)));
      if (!chunks.empty()) {
        SV_TRY(d_chunks.alloc(chunks.size()));
        SV_TRY(rcb.add_h2d(d_chunks.get(), chunks));
      }
      SV_TRY(rcb.flush());
      PhaseTimer tm(c, SIEVE_PHASE_SORT, nin * 8);
      launch_grid_tab(segs.get(), nseg, G, gtab.get(), S);
      // the cell keys go where an odd number of radix passes ends in ck (no copy-back), and
      // k_cellkey accumulates the sort's digit histograms as it writes them (no histogram read)
      u64* ck_in = radix_sort_keys_input(ck.get(), nin, (int)ib, tmp.get());
      u32* ghist = (nin > 1 && ib <= 24) ? radix_sort_prepare(nin, false, (int)ib, tmp.get(), S) : nullptr;
      launch_cellkey(round == 1 ? nullptr : d_chunks.get(), src, nin, round == 1 ? bx : 64, src_shift,
                     segs.get(), G, gtab.get(), ib, (u32)ncell, s0, ck_in,
                     c->count_terms ? terms.get() : nullptr, ghist, S);
      int passes = 0;
      SV_TRY(radix_sort(ck.get(), nullptr, nin, (int)ib, tmp.get(), S, &passes, ck_in != ck.get(),
                        ghist != nullptr));
      if (c->timing) c->acc[SIEVE_PHASE_SORT].work += (u64)passes * nin * 16;
      launch_cell_offsets(ck.get(), nin, ib, (u32)ncell, off.get(), S);
      SV_CUDA(cudaGetLastError());
    }
    DBuf<u64> D(c);
    SV_TRY(D.alloc((size_t)nseg * G * 2));
    // part buffers (one rank: sized by the bound nseg * tstride, see below) are initialised with
    // the densities in one launch
    // Part slots: a guess of PART_GUESS parts per segment (never more than the bound
    // nseg * tstride), so neither the part moments nor their all-reduce wait for the host to learn
    // the part count; a round with more parts than slots redoes its part moments with the exact
    // count, which every rank reads after the round's one synchronisation (so all ranks agree).
    u32 cap = (u32)std::min<u64>((u64)nseg * tstride, (u64)nseg * PART_GUESS + 64);
    if (const char* e = getenv("SIEVE_PART_SLOTS"))  // test hook: force the exact-count redo
      cap = std::max<u32>(1, std::min<u32>(cap, (u32)atoi(e)));
    DBuf<u64> pl(c), pm(c), pab(c);
    SV_TRY(pl.alloc((size_t)cap * MOM_LANES));
    SV_TRY(pm.alloc((size_t)cap * 2));
    SV_TRY(pab.alloc((size_t)cap * 4));
    {
      FillRegions fr{{D.get(), pl.get(), pm.get(), pm.get() + cap},
                     {(u64)nseg * G * 2, (u64)cap * MOM_LANES, cap, cap}, {0, 0, ~0ull, 0}, 4};
      launch_fill_multi(fr, S);
    }
    if (nin) {
      DBuf<char> regions(c);
      DBuf<u32> tile_items(c);
      DBuf<char> stemp(c);
      SV_TRY(regions.alloc(kde_region_bytes((u64)nseg * tps)));
      SV_TRY(tile_items.alloc((size_t)nseg * tps + 1));
      SV_TRY(stemp.alloc(scan_u32_temp_bytes((u64)nseg * tps)));
      // work items are counted on the device; size the item map by a host-side bound so no
      // synchronisation is needed here: a tile has at most ceil(segment values / KDE_CH) + slack
      // items (its regions are disjoint runs of the segment's values)
      u64 items_bound = 0, global_bound = 0;
      for (u32 s = 0; s < nseg; s++) {
        u64 len = round == 1 ? h_localn[op[s].kid] : op[s].e - op[s].b;
        items_bound += (u64)tps * ((len + KDE_CH - 1) / KDE_CH + kde_items_per_tile_slack());
        global_bound += (u64)tps * ((op[s].n + KDE_CH - 1) / KDE_CH + kde_items_per_tile_slack());  // replicated
      }
      // the limit is decided on the segments' GLOBAL counts, identical on every rank, so no rank
      // returns while the others enter AR-2 (the local bound is at most the global one)
      if (global_bound >= (1ull << 32)) return sv_fail(SIEVE_ELIMIT, "too many KDE work items");
      u32 items = (u32)items_bound;
      DBuf<char> item_tile(c);
      SV_TRY(item_tile.alloc(kde_item_bytes(items)));
      {
        PhaseTimer tp(c, SIEVE_PHASE_KDE_PLAN, 0);
        kde_plan(segs.get(), nseg, G, gtab.get(), off.get(), regions.get(), tile_items.get(), stemp.get(),
                 item_tile.get(), S);
      }
      PhaseTimer tm(c, SIEVE_PHASE_KDE, 0);
      // the unguarded KDE variant needs |z| < 4800 for every evaluated pair: window 7.6 h plus
      // KDE_TJ - 1 grid steps plus two boundary cells, so max Delta / h < 140 suffices
      bool guard = false;
      for (u32 s = 0; s < nseg; s++)
        if ((double)(hs[s].hi - hs[s].lo) / (double)(G - 1) >= 140.0 * hs[s].h) guard = true;
      launch_kde(segs.get(), nseg, G, ck.get(), vsh, regions.get(), tile_items.get(),
                 item_tile.get(), items, D.get(), terms.get() + 1, guard, false, S);
      tm.stop();
      SV_CUDA(cudaGetLastError());
      if (getenv("SIEVE_KDE_STATS")) {  // diagnostic: work items of this round
        const u64 nt = (u64)nseg * tps;
        std::vector<u32> hi(nt + 1);
        SV_CUDA(cudaStreamSynchronize(S));
        SV_CUDA(cudaMemcpy(hi.data(), tile_items.get(), 4 * (nt + 1), cudaMemcpyDeviceToHost));
        fprintf(stderr, "[kde stats] round=%u nseg=%u tiles=%llu items=%u\n", round, nseg,
                (unsigned long long)nt, hi[nt]);
      }
    }
    // AR-2: the densities' two u64 lanes per grid point (16 B), summed as the KDE left them;
    // k_valleys normalises them to u128
    if (c->comm) SV_TRY(allreduce(c, D.get(), (size_t)nseg * G * 2, RED_SUM));
    DBuf<u64> T(c);
    DBuf<u32> ntk(c), d_off(c);
    SV_TRY(T.alloc((size_t)nseg * tstride));
    SV_TRY(ntk.alloc((size_t)nseg * 2));
    SV_TRY(d_off.alloc(nseg + 1));
    PhaseTimer tv(c, SIEVE_PHASE_REFINE, 0);
    launch_valleys(segs.get(), nseg, G, P->valley_shift, D.get(), T.get(), tstride, ntk.get(),
                   ntk.get() + nseg, R->keep_debug, S);
    launch_part_offsets(ntk.get(), nseg, d_off.get(), S);
    tv.stop();
    // Part moments (AR-3 as one grouped step: SUM of the limb lanes, MAX of the complemented
    // mins and of the maxes), packed into mapped host memory: ONE host synchronisation per round
    // at any rank count.
    std::vector<u32> h_ntk(2 * (size_t)nseg);   // cut counts and split kinds, from the part records
    std::vector<u64> h_D, h_T;
    if (R->keep_debug) {
      CopyBatch ecb(c);   // read back with the part records at the round's synchronisation
      SV_TRY(ecb.add_d2h(h_D, D.get(), (size_t)nseg * G * 2));
      SV_TRY(ecb.add_d2h(h_T, T.get(), (size_t)nseg * tstride));
      SV_TRY(ecb.flush());
    }
    u64 *hrec = nullptr, *drec = nullptr;
    for (int pass = 0;; pass++) {
      DBuf<u32> pitems(c);
      DBuf<char> ptemp(c);
      SV_TRY(pitems.alloc(cap + 1));
      SV_TRY(ptemp.alloc(scan_u32_temp_bytes(cap)));
      {
        PhaseTimer tp(c, SIEVE_PHASE_REFINE, 0);
        launch_part_stats(segs.get(), nseg, G, gtab.get(), off.get(), T.get(), tstride, ntk.get(), d_off.get(),
                          cap, ck.get(), vsh, pitems.get(), ptemp.get(), pl.get(), pm.get(), pab.get(), S);
        SV_CUDA(cudaGetLastError());
      }
      if (c->comm) {
        launch_complement(pm.get(), cap, 1, S);
        SV_TRY(allreduce_group(c, {{pl.get(), (size_t)cap * MOM_LANES, RED_SUM}, {pm.get(), (size_t)cap * 2, RED_MAX}}));
        launch_complement(pm.get(), cap, 1, S);
      }
      SV_TRY(mapped_get(c, (int)(nbatch & 1), (1 + (size_t)cap * PART_REC + nseg) * 8, &hrec, &drec));
      launch_part_pack(d_off.get(), nseg, cap, pl.get(), pm.get(), pab.get(), ntk.get(), P->theta_num,
                       P->theta_den, drec, S);
      hc.mark("p");
      take_finals();   // the previous batch's, while this one runs
      hc.mark("fin");
      SV_TRY(sync(c));
      hc.mark("ps");
      const u64 live = hrec[0];  // replicated: every rank computed the same cuts from the same D
      for (u32 q = 0; q < nseg; q++) {
        const u64 w = hrec[1 + (size_t)cap * PART_REC + q];
        h_ntk[q] = (u32)w;
        h_ntk[nseg + q] = (u32)(w >> 32);
      }
      if (live <= cap) break;
      if (pass > 0) return sv_fail(SIEVE_ESTATE, "internal: part count grew");
      cap = (u32)live;  // more parts than slots: redo this round's part moments with the exact count
      SV_TRY(pl.alloc((size_t)cap * MOM_LANES));
      SV_TRY(pm.alloc((size_t)cap * 2));
      SV_TRY(pab.alloc((size_t)cap * 4));
      FillRegions fr{{pl.get(), pm.get(), pm.get() + cap, nullptr},
                     {(u64)cap * MOM_LANES, cap, cap, 0}, {0, ~0ull, 0, 0}, 3};
      launch_fill_multi(fr, S);
    }
    std::vector<u32> part_off(nseg + 1);
    u32 nparts = 0;
    for (u32 s = 0; s < nseg; s++) { part_off[s] = nparts; nparts += h_ntk[s] + 1; }
    part_off[nseg] = nparts;
    if (hrec[0] != nparts) return sv_fail(SIEVE_ESTATE, "internal: part count mismatch");
    hc.mark("rec");
    nbatch++;
    if (rec) {   // the sweep's tree: this batch's segments' bandwidths, parts and re-opened children
      for (u32 q = 0; q < nseg; q++) {
        SweepTree::Seg& g = rec->segs[op[q].node];
        g.h = hh[q];
        g.p0 = (u32)rec->parts.size();
        for (u32 p = part_off[q]; p < part_off[q + 1]; p++) {
          const u64* L = hrec + 1 + (size_t)p * PART_REC;
          if (!L[0]) continue;
          rec->parts.push_back({L[MOM_LANES], L[MOM_LANES + 1], L[0], limbs_u128(L + 1), limbs_u128(L + 5), -1});
        }
        g.p1 = (u32)rec->parts.size();
      }
    }
    {
      DeferredFin d;
      d.rec = hrec;
      d.round = round;
      d.part_off = part_off;
      d.kid.resize(nseg);
      for (u32 q = 0; q < nseg; q++) d.kid[q] = op[q].kid;
      d.h.assign(hh.begin(), hh.end());
      dfin.push_back(std::move(d));
    }
    for (u32 s = 0; s < nseg; s++) {
      if (R->keep_debug) {
        SegDebug sd;
        sd.meta.kernel_id = op[s].kid;
        sd.meta.round = round;
        sd.meta.split_kind = h_ntk[nseg + s];
        sd.meta.n_cuts = h_ntk[s];
        sd.meta.lo = op[s].lo;
        sd.meta.hi = op[s].hi;
        sd.meta.count = op[s].n;
        sd.meta.bandwidth = hh[s];
        sd.dlo.resize(G); sd.dhi.resize(G);
        for (u32 j = 0; j < G; j++) {
          sd.dlo[j] = h_D[2 * ((size_t)s * G + j)];
          sd.dhi[j] = h_D[2 * ((size_t)s * G + j) + 1];
        }
        sd.cuts.assign(h_T.begin() + (size_t)s * tstride, h_T.begin() + (size_t)s * tstride + h_ntk[s]);
        R->segs.push_back(std::move(sd));
      }
      for (u32 p = part_off[s]; p < part_off[s + 1]; p++) {
        const u64* L = hrec + 1 + (size_t)p * PART_REC;  // {lanes[9], min, max, ia, ib, final}
        // empty parts are dropped (A13 f); final parts go to the strata later (take_finals);
        // a re-opened part's values are [ia, ib) of this batch's grouped values
        if (L[0] && !L[MOM_LANES + 4]) {
          next.push_back({op[s].kid, op[s].t3rank, L[MOM_LANES], L[MOM_LANES + 1], L[0], limbs_u128(L + 1),
                          limbs_u128(L + 5), L[MOM_LANES + 2], L[MOM_LANES + 3], ck.get(), vsh});
          if (rec) {   // the re-opened part's segment node (its part record is the p-th non-empty)
            const int node = (int)rec->segs.size();
            next.back().node = node;
            rec->segs.push_back({op[s].kid, round + 1, L[MOM_LANES], L[MOM_LANES + 1], L[0], limbs_u128(L + 1),
                                 limbs_u128(L + 5), 0.0, 0, 0});
            u32 pi = rec->segs[op[s].node].p0;
            for (u32 p2 = part_off[s]; p2 < p; p2++) pi += hrec[1 + (size_t)p2 * PART_REC] != 0;
            rec->parts[pi].child = node;
          }
        }
      }
    }
    }  // batches
    open.swap(next);
    hc.mark("round");
  }
  take_finals();   // the last batch's
  R->rounds = use ? use_rounds : round;
  // the KDE term count is read back with the representatives at the end (no extra sync)
  std::vector<unsigned long long> h_terms;
  keys.release();
  hc.mark("rend");

  // ---------------- stratum table: order by (kernel, lo) (A23) --------------------------------
  // One pass: the Tier-1/2 strata (one per kernel, in kernel order) merged with the sorted Tier-3
  // strata (disjoint kernels), building the permutation, the per-kernel lookup table, the lower
  // bounds, the tiers and the weights together.
  const u32 ns = (u32)fin.size();
  static thread_local std::vector<u32> order_tl;
  std::vector<u32>& order = order_tl;
  order.resize(ns);
  auto F = [&](u32 s) -> const Fin& { return fin[order[s]]; };
  // the call's host tables keep their capacity across calls (no allocation or first-touch page
  // faults between the last round's synchronisation and pass B's launch)
  static thread_local std::vector<KTab> ktab_tl;
  static thread_local std::vector<u64> lows_tl, hW_tl;
  static thread_local std::vector<u32> tiers_tl;
  std::vector<KTab>& ktab = ktab_tl;
  std::vector<u64>& lows = lows_tl;
  std::vector<u32>& tiers = tiers_tl;
  std::vector<u64>& hW = hW_tl;
  ktab.assign(K, KTab{0, 0, 0, 0});
  lows.clear();
  tiers.resize(ns);
  hW.resize(2 * (size_t)ns);
  {
    u32 i = 0, s = 0;
    size_t j = 0;
    while (i < n12 || j < t3s.size()) {
      const u32 idx = (j == t3s.size() || (i < n12 && fin[i].kid < (u32)(t3s[j].first >> 44))) ? i++ : t3s[j++].second;
      const Fin& f = fin[idx];
      order[s] = idx;
      tiers[s] = f.tier;
      KTab& e = ktab[f.kid];
      if (e.m == 0) { e.base = s; e.lows_off = (u32)lows.size(); }
      else lows.push_back(f.lo);   // a kernel's strata 1..m-1 lower bounds, contiguous, ascending
      e.m++;
      hW[2 * (size_t)s] = (u64)f.s1;
      hW[2 * (size_t)s + 1] = (u64)(f.s1 >> 64);
      s++;
    }
    if (s != ns) return sv_fail(SIEVE_ESTATE, "internal: stratum order");
  }
  if (lows.empty()) lows.push_back(0);

  hc.mark("table");
  // ---------------- pass B: assignment + (stratum, CTA) statistics ---------------------
  DBuf<KTab> d_ktab(c);
  DBuf<u64> d_lows(c), errf(c);
  SV_TRY(d_ktab.alloc(K));
  SV_TRY(d_lows.alloc(lows.size()));
  SV_TRY(errf.alloc(4));
  // the strata weights W_s = S1_s (u128) on the device for the prediction computed with the
  // representatives (below), uploaded with the assignment tables
  DBuf<u64> dW(c);
  DBuf<double> dpred(c);
  SV_TRY(dW.alloc(std::max<size_t>(hW.size(), 2)));
  SV_TRY(dpred.alloc(4));
  {
    CopyBatch cb(c);
    SV_TRY(cb.add_h2d(d_ktab.get(), ktab));
    SV_TRY(cb.add_h2d(d_lows.get(), lows));
    SV_TRY(cb.add_h2d(dW.get(), hW));
    SV_TRY(cb.flush());
  }
  std::vector<double> h_pred;
  u64 cap = 1;
  while (cap < std::max<u64>(1u << 16, 8ull * ns)) cap <<= 1;
  // One rank: the (stratum, CTA) entries go to the representatives without a host round trip --
  // the compacted arrays are pre-filled with neutral entries (key ~0 sorts last, count 0), so
  // every later launch can be sized by the table capacity; the overflow flag is read with the
  // representatives (one synchronisation) and an overflow redoes pass B with a bigger table.
  // Several ranks: the entry counts are exchanged first (AR-4 needs them on the host).
  std::vector<u64> h_rep, h_xy, hflag;
  // the stratum table's fields that do not depend on the representatives, filled while pass B
  // and the representatives run (the rest after the synchronisation)
  bool table_pre = false;
  auto assemble_pre = [&]() {
    R->st.swap(spare_strata());   // capacity from a freed result of this thread (no page faults)
    R->st.resize(ns);               // value-initialised: every field is set, the pad is zero
    static thread_local std::vector<u32> first_of_tl;
    std::vector<u32>& first_of = first_of_tl;
    first_of.assign(K, 0xFFFFFFFFu);
    for (u32 s = 0; s < ns; s++) {
      const Fin& f = F(s);
      sieve_stratum& o = R->st[s];
      if (first_of[f.kid] == 0xFFFFFFFFu) first_of[f.kid] = s;
      o.kernel_id = f.kid;
      o.tier = f.tier;
      o.index_in_kernel = s - first_of[f.kid];
      o.lo = f.lo; o.hi = f.hi; o.count = f.n;
      o.instr_sum_lo = (u64)f.s1; o.instr_sum_hi = (u64)(f.s1 >> 64);
      o.bandwidth = f.h;
      o.split_round = f.round;
    }
    table_pre = true;
  };
  for (int attempt = 0;; attempt++) {
    if (attempt > 6) return sv_fail(SIEVE_ENOMEM, "(stratum, CTA) table kept overflowing");
    DBuf<u64> gkeys(c), gcnt(c), gfirst(c), ent(c);
    SV_TRY(gkeys.alloc(cap)); SV_TRY(gcnt.alloc(cap)); SV_TRY(gfirst.alloc(cap));
    SV_TRY(ent.alloc(cap * 3));   // [keys | counts | firsts] of the compacted entries
    {  // every initialisation of pass B in two launches (the table, then the entry arrays)
      FillRegions f1{{gkeys.get(), gcnt.get(), gfirst.get(), errf.get()}, {cap, cap, cap, 4},
                     {HASH_EMPTY, 0, ~0ull, 0}, 4};
      launch_fill_multi(f1, S);
      FillRegions f2{{ent.get(), ent.get() + cap, ent.get() + 2 * cap, (u64*)counter.get()}, {cap, cap, cap, 1},
                     {~0ull, 0, ~0ull, 0}, 4};
      launch_fill_multi(f2, S);
    }
    GHash gh{gkeys.get(), gcnt.get(), gfirst.get(), cap};
    {
      PhaseTimer tb(c, SIEVE_PHASE_ASSIGN, n * (12 + (t->cta ? 4 : 0) + (sid_out ? 4 : 0)));
      launch_assign(t->kid, t->x, t->cta, n, t->first_id, d_ktab.get(), d_lows.get(), K,
                    (u32)lows.size(), ns, sid_out, gh, errf.get(), assign_grid(), S);
    }
    SV_CUDA(cudaGetLastError());
    launch_hash_compact(gh, ent.get(), ent.get() + cap, ent.get() + 2 * cap, counter.get(), S);
    u64 Etot = cap;
    const u64* ak = ent.get();
    DBuf<u64> akb(c);
    if (c->comm) {
      // one exchange of world + 1 lanes (SUM) and ONE synchronisation: [0] = ranks whose table
      // overflowed (the retry decision is then identical on every rank), [1 + r] = rank r's
      // entry count (the offsets of the all-gather below)
      DBuf<u64> xw(c);
      SV_TRY(xw.alloc((size_t)c->world + 1));
      launch_exchange_prep(errf.get() + 2, counter.get(), c->comm->rank, c->world, xw.get(), S);
      SV_TRY(allreduce(c, xw.get(), (size_t)c->world + 1, RED_SUM));
      std::vector<u64> all;
      SV_TRY(d2h(c, all, xw.get(), (size_t)c->world + 1));
      SV_TRY(sync(c));
      if (all[0]) { cap <<= 2; continue; }
      const u64 E = all[1 + c->rank];
      // gather every rank's entries (AR-4: all-gather expressed as a SUM over zero-padded slots)
      Etot = 0;
      u64 Eoff = 0;
      for (int r = 0; r < c->world; r++) { if (r == c->rank) Eoff = Etot; Etot += all[1 + r]; }
      SV_TRY(akb.alloc(std::max<u64>(Etot, 1) * 3));
      SV_CUDA(cudaMemsetAsync(akb.get(), 0, Etot * 3 * 8, S));
      SV_CUDA(cudaMemcpyAsync(akb.get() + Eoff, ent.get(), E * 8, cudaMemcpyDeviceToDevice, S));
      SV_CUDA(cudaMemcpyAsync(akb.get() + Etot + Eoff, ent.get() + cap, E * 8, cudaMemcpyDeviceToDevice, S));
      SV_CUDA(cudaMemcpyAsync(akb.get() + 2 * Etot + Eoff, ent.get() + 2 * cap, E * 8, cudaMemcpyDeviceToDevice, S));
      SV_TRY(allreduce(c, akb.get(), Etot * 3, RED_SUM));
      ak = akb.get();
    }
    hc.mark("passB");
    // sort entries by (stratum, CTA) with their index as payload, then gather count / first;
    // nbits covers every stratum id with a spare bit, so a neutral key (~0) sorts last
    DBuf<u32> idx(c);
    DBuf<u64> sk(c), scnt(c), sfirst(c);
    SV_TRY(idx.alloc(std::max<u64>(Etot, 1)));
    SV_TRY(sk.alloc(std::max<u64>(Etot, 1))); SV_TRY(scnt.alloc(std::max<u64>(Etot, 1)));
    SV_TRY(sfirst.alloc(std::max<u64>(Etot, 1)));
    launch_iota_u32(idx.get(), Etot, S);
    PhaseTimer tr(c, SIEVE_PHASE_REPS, 0);
    if (c->comm) {  // equal (stratum, CTA) keys from several ranks must end up adjacent
      launch_copy(sk.get(), ak, Etot * 8, S);
      DBuf<char> tmp(c);
      SV_TRY(tmp.alloc(radix_sort_temp_bytes(Etot, true, 32 + (int)bitlen(ns))));
      SV_TRY(radix_sort(sk.get(), idx.get(), Etot, 32 + (int)bitlen(ns), tmp.get(), S));
    } else {
      // one rank: every (stratum, CTA) key occurs once, so grouping by stratum suffices (the
      // dominant CTA and the first invocation do not depend on the order within a stratum):
      // sort the stratum ids alone (neutral slots map to ns and sort last), then gather the keys
      DBuf<u64> sid(c);
      SV_TRY(sid.alloc(std::max<u64>(Etot, 1)));
      launch_entry_sids(ak, Etot, ns, sid.get(), S);
      DBuf<char> tmp(c);
      SV_TRY(tmp.alloc(radix_sort_temp_bytes(Etot, true, (int)bitlen(ns))));
      SV_TRY(radix_sort(sid.get(), idx.get(), Etot, (int)bitlen(ns), tmp.get(), S));
      launch_gather_u64(ak, idx.get(), Etot, sk.get(), S);
    }
    launch_gather_u64(ak + Etot, idx.get(), Etot, scnt.get(), S);
    launch_gather_u64(ak + 2 * Etot, idx.get(), Etot, sfirst.get(), S);
    DBuf<u32> d_tier(c);
    DBuf<u64> rep(c), repxy(c);
    SV_TRY(d_tier.alloc(ns));
    SV_TRY(rep.alloc(2 * (size_t)ns));
    SV_TRY(repxy.alloc(2 * (size_t)ns));
    {
      CopyBatch cb(c);
      SV_TRY(cb.add_h2d(d_tier.get(), tiers));
      SV_TRY(cb.flush());
    }
    launch_reps(sk.get(), scnt.get(), sfirst.get(), Etot, d_tier.get(), ns, rep.get(), rep.get() + ns, S);
    launch_rep_xy(rep.get(), ns, t->first_id, n, t->x, t->y, repxy.get(), S);
    tr.stop();
    SV_CUDA(cudaGetLastError());
    SV_TRY(allreduce(c, repxy.get(), 2 * (size_t)ns, RED_SUM));   // AR-5: owner contributes
    // the prediction from the trace's own cycles: the kernel and inputs
    // sieve_predict uses, computed here so it costs no extra synchronisation
    const bool pre_pred = t->y != nullptr && ns > 0;
    if (pre_pred) {
      PhaseTimer tpr(c, SIEVE_PHASE_PREDICT, 0);
      launch_predict(dW.get(), repxy.get(), repxy.get() + ns, ns, 1, dpred.get(), S);
    }
    {
      CopyBatch cb(c);
      SV_TRY(cb.add_d2h(h_rep, rep.get(), 2 * (size_t)ns));
      SV_TRY(cb.add_d2h(h_xy, repxy.get(), 2 * (size_t)ns));
      if (pre_pred) SV_TRY(cb.add_d2h(h_pred, dpred.get(), 4));
      if (!c->comm) SV_TRY(cb.add_d2h(hflag, errf.get(), 4));
      if (h_terms.empty()) SV_TRY(cb.add_d2h(h_terms, terms.get(), 2));
      SV_TRY(cb.flush());
    }
    if (!table_pre) assemble_pre();
    SV_TRY(sync(c));
    if (!c->comm && hflag[2]) { cap <<= 2; continue; }
    break;
  }
  resolve_timing(c);
  if (!h_pred.empty()) {
    R->pred_ok = true;
    R->pred_serial = t->serial;
    for (int i = 0; i < 4; i++) R->pred_r[i] = h_pred[i];
  }
  R->kde_terms = h_terms[0];
  R->kde_evaluated = h_terms[1];
  if (c->timing) c->acc[SIEVE_PHASE_KDE].work += h_terms[0];
  hc.mark("reps");
  struct AssembleMark { HostClock& h; ~AssembleMark() { h.mark("assemble"); } } assemble_mark{hc};

  // ---------------- assemble: the representatives' fields ---------------------------------------
  for (u32 s = 0; s < ns; s++) {
    sieve_stratum& o = R->st[s];
    o.rep_cta = (u32)h_rep[ns + s];
    o.rep_id = h_rep[s];
    o.rep_instr = h_xy[s];
    o.rep_cycles = h_xy[ns + (size_t)s];
  }
  return SIEVE_OK;
}

static int check_params(const sieve_params* p, sieve_params* P) {
  if (p) *P = *p; else sieve_params_default(P);
  if (P->theta_num == 0 || P->theta_den == 0) return sv_fail(SIEVE_EINVAL, "theta must be a positive fraction");
  if (P->grid_points < 3 || P->grid_points > 65536) return sv_fail(SIEVE_EINVAL, "grid_points must be in [3, 65536]");
  if (P->valley_shift > 120) return sv_fail(SIEVE_EINVAL, "valley_shift must be <= 120");
  if (!(P->bw_scale > 0)) return sv_fail(SIEVE_EINVAL, "bw_scale must be > 0");
  if (P->max_rounds == 0) P->max_rounds = 1;
  return SIEVE_OK;
}

static int stratify_one(sieve_trace t, const sieve_params* P, uint32_t* sid_out, sieve_strata* out,
                        const MomentsHost* cached, SweepTree* rec = nullptr, const SweepTree* use = nullptr) {
  sieve_ctx c = t->ctx;
  sieve_strata_s* R = new sieve_strata_s();
  R->ctx = c;
  R->G = P->grid_points;
  R->keep_debug = P->keep_debug != 0;
  R->has_cycles = t->y != nullptr;
  int st = stratify_impl(t, P, sid_out, R, cached, rec, use);
  if (st != SIEVE_OK) {
    cudaStreamSynchronize(c->stream);
    delete R;
    return st;
  }
  *out = R;
  return SIEVE_OK;
}

extern "C" int sieve_stratify(sieve_trace t, const sieve_params* p, uint32_t* sid_out, sieve_strata* out) {
  if (!out) return sv_fail(SIEVE_EINVAL, "out is NULL");
  *out = nullptr;
  if (!trace_ok(t)) return sv_fail(SIEVE_EINVAL, "bad trace handle");
  sieve_params P;
  SV_TRY(check_params(p, &P));
  SV_CUDA(cudaSetDevice(t->ctx->device));
  return stratify_one(t, &P, sid_out, out, nullptr);
}

extern "C" int sieve_stratify_sweep(sieve_trace t, const sieve_params* p, uint32_t count,
                                    const uint32_t* theta_num, const uint32_t* theta_den,
                                    sieve_strata* outs) {
  if (!outs || (count && (!theta_num || !theta_den))) return sv_fail(SIEVE_EINVAL, "NULL argument");
  for (uint32_t i = 0; i < count; i++) outs[i] = nullptr;
  if (!trace_ok(t)) return sv_fail(SIEVE_EINVAL, "bad trace handle");
  sieve_params P;
  SV_TRY(check_params(p, &P));
  for (uint32_t i = 0; i < count; i++)
    if (!theta_num[i] || !theta_den[i]) return sv_fail(SIEVE_EINVAL, "theta must be a positive fraction");
  sieve_ctx c = t->ctx;
  SV_CUDA(cudaSetDevice(c->device));
  SV_TRY(arena_reset(c));
  MomentsHost M;
  SV_TRY(moments_pass(t, &M));  // pass A once for every theta
  // The refinement runs once, at the smallest theta, recording its tree; every other theta takes
  // the tree's frontier (SweepTree) and runs only the tiers, the table and pass B.  keep_debug
  // (every KDE segment of each theta's own refinement) and the SIEVE_SWEEP_SEPARATE test hook
  // refine every theta separately.
  const bool tree = count > 1 && !P.keep_debug && !getenv("SIEVE_SWEEP_SEPARATE");
  uint32_t imin = 0;
  for (uint32_t i = 1; i < count; i++)   // theta_i < theta_min, exactly
    if ((u64)theta_num[i] * theta_den[imin] < (u64)theta_num[imin] * theta_den[i]) imin = i;
  SweepTree T;
  T.root.assign(t->K, -1);
  auto run = [&](uint32_t i, SweepTree* rec, const SweepTree* use) {
    P.theta_num = theta_num[i];
    P.theta_den = theta_den[i];
    return stratify_one(t, &P, nullptr, &outs[i], &M, rec, use);
  };
  auto fail = [&](int st) {
    for (uint32_t j = 0; j < count; j++) { if (outs[j]) sieve_strata_free(outs[j]); outs[j] = nullptr; }
    return st;
  };
  if (tree) {
    int st = run(imin, &T, nullptr);
    if (st != SIEVE_OK) return fail(st);
  }
  for (uint32_t i = 0; i < count; i++) {
    if (tree && i == imin) continue;
    int st = run(i, nullptr, tree ? &T : nullptr);
    if (st != SIEVE_OK) return fail(st);
  }
  return SIEVE_OK;
}

extern "C" int sieve_tier_census(sieve_trace t, uint32_t count, const uint32_t* theta_num,
                                 const uint32_t* theta_den, uint64_t* kernels, uint64_t* invocations,
                                 uint64_t* instructions) {
  if (!trace_ok(t) || (count && (!theta_num || !theta_den || !kernels || !invocations)))
    return sv_fail(SIEVE_EINVAL, "bad argument");
  for (uint32_t i = 0; i < count; i++)
    if (!theta_num[i] || !theta_den[i]) return sv_fail(SIEVE_EINVAL, "theta must be a positive fraction");
  sieve_ctx c = t->ctx;
  SV_CUDA(cudaSetDevice(c->device));
  SV_TRY(arena_reset(c));
  MomentsHost M;
  SV_TRY(moments_pass(t, &M));
  for (uint32_t i = 0; i < count; i++) {
    u64 nk[3] = {0, 0, 0}, ni[3] = {0, 0, 0};
    u128 ins[3] = {0, 0, 0};
    for (u32 k = 0; k < t->K; k++) {
      const u64* L = &M.lanes[(size_t)k * MOM_LANES];
      if (!L[0]) continue;
      u128 s1 = limbs_u128(L + 1), s2 = limbs_u128(L + 5);
      int tier = M.mm[2 * k] == M.mm[2 * k + 1] ? 0 : (cov_lt(L[0], s1, s2, theta_num[i], theta_den[i]) ? 1 : 2);
      nk[tier]++;
      ni[tier] += L[0];
      ins[tier] += s1;
    }
    for (int j = 0; j < 3; j++) {
      kernels[3 * (size_t)i + j] = nk[j];
      invocations[3 * (size_t)i + j] = ni[j];
      if (instructions) {
        instructions[6 * (size_t)i + 2 * j] = (u64)ins[j];
        instructions[6 * (size_t)i + 2 * j + 1] = (u64)(ins[j] >> 64);
      }
    }
  }
  return SIEVE_OK;
}

// ------------------------------------------------------------------------------------------
// sieve_min_strata: the exact optimum of P:89's "(1)" (NEXT-3, reading A28)
// ------------------------------------------------------------------------------------------
extern "C" int sieve_min_strata(sieve_trace t, uint32_t theta_num, uint32_t theta_den,
                                uint32_t max_distinct, uint32_t* counts, uint64_t* cuts,
                                uint64_t cuts_cap, uint64_t* n_cuts) {
  if (!trace_ok(t) || !counts) return sv_fail(SIEVE_EINVAL, "bad argument");
  if (!theta_num || !theta_den) return sv_fail(SIEVE_EINVAL, "theta must be a positive fraction");
  sieve_ctx c = t->ctx;
  if (c->comm) return sv_fail(SIEVE_ESTATE, "sieve_min_strata is a single-rank diagnostic");
  cudaStream_t S = c->stream;
  SV_CUDA(cudaSetDevice(c->device));
  SV_TRY(arena_reset(c));
  MomentsHost M;
  SV_TRY(moments_pass(t, &M));
  const u32 K = t->K;
  std::vector<u32> t3rank(K, 0xFFFFFFFFu), t3kid;
  u64 n3 = 0;
  for (u32 k = 0; k < K; k++) {
    const u64* L = &M.lanes[(size_t)k * MOM_LANES];
    counts[k] = 0;
    if (!L[0]) continue;
    counts[k] = 1;
    if (M.mm[2 * k] == M.mm[2 * k + 1] || cov_lt(L[0], limbs_u128(L + 1), limbs_u128(L + 5), theta_num, theta_den))
      continue;  // Tier-1/2: one valid stratum
    t3rank[k] = (u32)t3kid.size();
    t3kid.push_back(k);
    n3 += L[0];
  }
  const u32 nk = (u32)t3kid.size();
  u64 total = 0;
  std::vector<u64> h_cuts;
  if (nk) {
    const u32 bx = std::max<u32>(1, bitlen(M.tot[4]));
    const u64 xmask = (bx >= 64) ? ~0ull : ((1ull << bx) - 1);
    const int nbits = (int)(bx + bitlen(nk - 1));
    DBuf<u64> keys(c);
    DBuf<u32> d_t3rank(c), flag(c), seg(c);
    DBuf<unsigned long long> counter(c);
    SV_TRY(counter.alloc(1));
    SV_TRY(d_t3rank.alloc(K));
    SV_TRY(h2d(c, d_t3rank.get(), t3rank));
    SV_TRY(keys.alloc(n3));
    SV_CUDA(cudaMemsetAsync(counter.get(), 0, 8, S));
    launch_t3_compact(t->kid, t->x, t->n, d_t3rank.get(), bx, keys.get(), counter.get(), S);
    {
      DBuf<char> tmp(c);
      SV_TRY(tmp.alloc(radix_sort_temp_bytes(n3, false, nbits)));
      SV_TRY(radix_sort(keys.get(), nullptr, n3, nbits, tmp.get(), S));
    }
    // run-length encoding: distinct keys, run starts, Tier-3 rank starts
    DBuf<char> stemp(c);
    SV_TRY(flag.alloc(n3)); SV_TRY(seg.alloc(n3 + 1)); SV_TRY(stemp.alloc(scan_u32_temp_bytes(n3)));
    launch_csv_heads(keys.get(), n3, flag.get(), S);
    scan_u32(flag.get(), seg.get(), n3, stemp.get(), seg.get() + n3, S);
    std::vector<u32> h_nu;
    SV_TRY(d2h(c, h_nu, seg.get() + n3, 1));
    SV_TRY(sync(c));
    const u64 nu = h_nu[0];
    DBuf<u64> ukey(c), Pn(c), dcuts(c), doff(c), out(c);
    DBuf<u32> ustart(c), kstart(c), f(c), arg(c), dcount(c);
    DBuf<u128> P1(c), P2(c);
    SV_TRY(ukey.alloc(nu)); SV_TRY(ustart.alloc(nu + 1)); SV_TRY(kstart.alloc(nk + 1));
    SV_TRY(Pn.alloc(nu + nk)); SV_TRY(P1.alloc(nu + nk)); SV_TRY(P2.alloc(nu + nk));
    SV_TRY(f.alloc(nu + nk)); SV_TRY(arg.alloc(nu + nk)); SV_TRY(dcount.alloc(nk)); SV_TRY(dcuts.alloc(nu));
    std::vector<u32> ends = {(u32)n3};
    std::vector<u32> kend = {(u32)nu};
    SV_TRY(h2d(c, ustart.get() + nu, ends));
    SV_TRY(h2d(c, kstart.get() + nk, kend));
    launch_rle(keys.get(), flag.get(), seg.get(), n3, bx, ukey.get(), ustart.get(), kstart.get(), S);
    const u32 cap = max_distinct ? max_distinct : 16384u;
    // the DP by layers (dp.cu): layer k assigns f(j) = k; one synchronisation per layer reads how
    // many kernels still lack f(m) (the layers number the largest optimum, not the values)
    DBuf<u32> la(c), lb(c), ca(c), cb(c), dstate(c), rem(c);
    SV_TRY(la.alloc(nu + nk)); SV_TRY(lb.alloc(nu + nk)); SV_TRY(ca.alloc(nk)); SV_TRY(cb.alloc(nk));
    SV_TRY(dstate.alloc(nk)); SV_TRY(rem.alloc(1));
    launch_dp_prefix(ukey.get(), ustart.get(), kstart.get(), nk, xmask, theta_num, theta_den, cap, Pn.get(),
                     P1.get(), P2.get(), f.get(), dcount.get(), la.get(), ca.get(), dstate.get(), S);
    u32* lst[2] = {la.get(), lb.get()};
    u32* lct[2] = {ca.get(), cb.get()};
    for (u32 k = 1;; k++) {
      if (k > nu + 1) return sv_fail(SIEVE_ESTATE, "internal: min-strata layers did not converge");
      SV_CUDA(cudaMemsetAsync(rem.get(), 0, 4, S));
      launch_dp_layer(kstart.get(), nk, (u32)nu, k, theta_num, theta_den, Pn.get(), P1.get(), P2.get(), f.get(),
                      arg.get(), lst[(k - 1) & 1], lct[(k - 1) & 1], dstate.get(), S);
      launch_dp_compact(kstart.get(), nk, k, f.get(), arg.get(), ukey.get(), xmask, lst[k & 1], lct[k & 1],
                        dstate.get(), dcount.get(), dcuts.get(), rem.get(), S);
      std::vector<u32> h_rem;
      SV_TRY(d2h(c, h_rem, rem.get(), 1));
      SV_TRY(sync(c));
      if (h_rem[0] == 0) break;
    }
    std::vector<u32> h_count;
    SV_TRY(d2h(c, h_count, dcount.get(), nk));
    SV_TRY(sync(c));
    SV_CUDA(cudaGetLastError());
    std::vector<u64> off(nk);
    for (u32 r = 0; r < nk; r++) {
      off[r] = total;
      counts[t3kid[r]] = h_count[r];
      if (h_count[r] >= 2 && h_count[r] != 0xFFFFFFFFu) total += h_count[r] - 1;
    }
    if (cuts && total && total <= cuts_cap) {
      SV_TRY(doff.alloc(nk)); SV_TRY(out.alloc(total));
      SV_TRY(h2d(c, doff.get(), off));
      launch_dp_gather(kstart.get(), dcount.get(), doff.get(), dcuts.get(), nk, out.get(), S);
      SV_TRY(d2h_raw(c, cuts, out.get(), total * 8));
      SV_TRY(sync(c));
    }
  }
  if (n_cuts) *n_cuts = total;
  if (cuts && total > cuts_cap) return sv_fail(SIEVE_ERANGE, "cuts_cap is smaller than *n_cuts");
  return SIEVE_OK;
}

extern "C" int sieve_strata_count(sieve_strata s, uint64_t* n) {
  if (!strata_ok(s) || !n) return sv_fail(SIEVE_EINVAL, "bad strata handle");
  *n = s->st.size();
  return SIEVE_OK;
}
extern "C" int sieve_strata_copy(sieve_strata s, sieve_stratum* host_out, uint64_t cap) {
  if (!strata_ok(s) || (!host_out && cap)) return sv_fail(SIEVE_EINVAL, "bad strata handle");
  u64 m = std::min<u64>(cap, s->st.size());
  if (m) memcpy(host_out, s->st.data(), m * sizeof(sieve_stratum));
  return SIEVE_OK;
}
extern "C" int sieve_strata_stats(sieve_strata s, uint32_t* rounds, uint64_t* terms,
                                  uint64_t* evaluated) {
  if (!strata_ok(s)) return sv_fail(SIEVE_EINVAL, "bad strata handle");
  if (rounds) *rounds = s->rounds;
  if (terms) *terms = s->kde_terms;
  if (evaluated) *evaluated = s->kde_evaluated;
  return SIEVE_OK;
}
extern "C" void sieve_strata_free(sieve_strata s) {
  if (!strata_ok(s)) return;
  s->magic = 0;
  std::vector<sieve_stratum>& sp = spare_strata();   // keep the larger buffer for the next result
  if (s->st.capacity() > sp.capacity()) { s->st.clear(); sp.swap(s->st); }
  delete s;
}
extern "C" int sieve_segment_count(sieve_strata s, uint64_t* n) {
  if (!strata_ok(s) || !n) return sv_fail(SIEVE_EINVAL, "bad strata handle");
  if (!s->keep_debug) return sv_fail(SIEVE_ESTATE, "stratify was called without keep_debug");
  *n = s->segs.size();
  return SIEVE_OK;
}
extern "C" int sieve_segment_get(sieve_strata s, uint64_t idx, sieve_segment* out, uint64_t* dlo,
                                 uint64_t* dhi, uint64_t* cuts) {
  if (!strata_ok(s)) return sv_fail(SIEVE_EINVAL, "bad strata handle");
  if (!s->keep_debug) return sv_fail(SIEVE_ESTATE, "stratify was called without keep_debug");
  if (idx >= s->segs.size()) return sv_fail(SIEVE_EINVAL, "segment index out of range");
  const SegDebug& d = s->segs[idx];
  if (out) *out = d.meta;
  if (dlo) memcpy(dlo, d.dlo.data(), d.dlo.size() * 8);
  if (dhi) memcpy(dhi, d.dhi.data(), d.dhi.size() * 8);
  if (cuts) memcpy(cuts, d.cuts.data(), d.cuts.size() * 8);
  return SIEVE_OK;
}

// ------------------------------------------------------------------------------------------
// sieve_predict
// ------------------------------------------------------------------------------------------
static double u128_to_double_host(u128 v) { return (double)v; }  // libgcc: correctly rounded

// ------------------------------------------------------------------------------------------
// sieve_cycle_cov: within-stratum cycle CoV (Fig. 4; reading A25: instruction
// weights for the average)
// ------------------------------------------------------------------------------------------
extern "C" int sieve_cycle_cov(sieve_strata s, sieve_trace t, const uint32_t* sid, double* cov,
                               double* weighted) {
  if (!strata_ok(s) || !trace_ok(t)) return sv_fail(SIEVE_EINVAL, "bad handle");
  if (!t->y) return sv_fail(SIEVE_EDOM, "the trace has no cycles column");
  if (t->n && !sid) return sv_fail(SIEVE_EINVAL, "stratum_of_invocation (device) is required");
  sieve_ctx c = t->ctx;
  SV_CUDA(cudaSetDevice(c->device));
  SV_TRY(arena_reset(c));
  const u32 ns = (u32)s->st.size();
  DBuf<char> part(c);
  DBuf<u64> lanes(c), errf(c);
  SV_TRY(part.alloc(group_moments_part_bytes(ns ? ns : 1)));
  SV_TRY(lanes.alloc((size_t)ns * GM_LANES));
  SV_TRY(errf.alloc(1));
  SV_CUDA(cudaMemsetAsync(errf.get(), 0, 8, c->stream));
  if (ns) launch_group_moments(sid, t->y, t->n, ns, (GMomPartial*)part.get(), lanes.get(), errf.get(), c->stream);
  SV_CUDA(cudaGetLastError());
  SV_TRY(allreduce(c, lanes.get(), (size_t)ns * GM_LANES, RED_SUM));
  SV_TRY(allreduce(c, errf.get(), 1, RED_MAX));
  std::vector<u64> h_l, h_e;
  SV_TRY(d2h(c, h_l, lanes.get(), (size_t)ns * GM_LANES));
  SV_TRY(d2h(c, h_e, errf.get(), 1));
  SV_TRY(sync(c));
  if (h_e[0]) return sv_fail(SIEVE_ERANGE, "cycle counts must be < 2^48 for sieve_cycle_cov");
  long double acc = 0, I = 0;
  for (u32 i = 0; i < ns; i++) {
    const u64* L = &h_l[(size_t)i * GM_LANES];
    u128 s1 = limbs_u128(L + 1);
    // S2 from 6 limb lanes (can exceed 2^128 across ranks)
    W256 s2 = {{0, 0, 0, 0}};
    {
      u128 carry = 0;
      u64 w32[8] = {0};
      for (int j = 0; j < 6; j++) {
        u128 v = (u128)L[5 + j] + carry;
        w32[j] = (u64)(v & 0xFFFFFFFFull);
        carry = v >> 32;
      }
      w32[6] = (u64)(carry & 0xFFFFFFFFull);
      w32[7] = (u64)(carry >> 32);
      for (int j = 0; j < 4; j++) s2.w[j] = w32[2 * j] | (w32[2 * j + 1] << 32);
    }
    double cv = 0.0;
    if (s1 != 0) {
      W256 d = w256_sub(w256_mul_small(s2, L[0]), w256_mul(s1, s1));
      cv = sqrt(w256_to_double(d)) / (double)s1;
    }
    if (cov) cov[i] = cv;
    long double W = (long double)(((u128)s->st[i].instr_sum_hi << 64) | s->st[i].instr_sum_lo);
    acc += W * cv;
    I += W;
  }
  if (weighted) *weighted = ns ? (double)(acc / I) : 0.0;
  return SIEVE_OK;
}

// M predictions at once: rep_cycles is [M][n_strata] (nullable iff M == 1: the trace's cycles)
static int predict_impl(sieve_strata s, sieve_trace t, u32 M, const uint64_t* rep_cycles,
                        sieve_prediction* out) {
  if (!strata_ok(s) || !trace_ok(t) || !out) return sv_fail(SIEVE_EINVAL, "bad handle");
  if (!rep_cycles && (M != 1 || !s->has_cycles))
    return sv_fail(SIEVE_EDOM, "no cycle source for the representatives");
  sieve_ctx c = t->ctx;
  SV_CUDA(cudaSetDevice(c->device));
  const u32 ns = (u32)s->st.size();
  std::vector<double> r;
  if (!rep_cycles && M == 1 && s->pred_ok && s->pred_serial == t->serial) {
    r.assign(s->pred_r, s->pred_r + 4);   // computed with the representatives (sieve_stratify)
  } else {
  SV_TRY(arena_reset(c));
  std::vector<u64> hW(2 * (size_t)ns), hx(ns), hy((size_t)M * ns);
  for (u32 i = 0; i < ns; i++) {
    hW[2 * i] = s->st[i].instr_sum_lo;
    hW[2 * i + 1] = s->st[i].instr_sum_hi;
    hx[i] = s->st[i].rep_instr;
  }
  for (u32 m = 0; m < M; m++)
    for (u32 i = 0; i < ns; i++)
      hy[(size_t)m * ns + i] = rep_cycles ? rep_cycles[(size_t)m * ns + i] : s->st[i].rep_cycles;
  DBuf<u64> dW(c), dx(c), dy(c);
  DBuf<double> dout(c);
  SV_TRY(dW.alloc(hW.size())); SV_TRY(dx.alloc(ns)); SV_TRY(dy.alloc(hy.size()));
  SV_TRY(dout.alloc(4 * (size_t)M));
  {
    CopyBatch cb(c);
    SV_TRY(cb.add_h2d(dW.get(), hW)); SV_TRY(cb.add_h2d(dx.get(), hx)); SV_TRY(cb.add_h2d(dy.get(), hy));
    SV_TRY(cb.flush());
  }
  PhaseTimer tpr(c, SIEVE_PHASE_PREDICT, 0);
  launch_predict(dW.get(), dx.get(), dy.get(), ns, M, dout.get(), c->stream);
  tpr.stop();
  SV_CUDA(cudaGetLastError());
  SV_TRY(d2h(c, r, dout.get(), 4 * (size_t)M));
  SV_TRY(sync(c));
  resolve_timing(c);
  }
  for (u32 m = 0; m < M; m++) {
    const double* rm = &r[4 * (size_t)m];
    sieve_prediction& o = out[m];
    o.predicted_cycles = rm[0];
    o.predicted_ipc = rm[3];
    o.total_instr_lo = (u64)s->total_instr;
    o.total_instr_hi = (u64)(s->total_instr >> 64);
    if (s->has_cycles) {
      double cm = u128_to_double_host(s->c_meas);
      o.measured_cycles = cm;
      o.error = s->c_meas == 0 ? NAN : fabs(rm[0] - cm) / cm;
      o.speedup = cm / rm[1];
    } else {
      o.measured_cycles = NAN;
      o.error = NAN;
      o.speedup = NAN;
    }
  }
  return SIEVE_OK;
}

extern "C" int sieve_predict(sieve_strata s, sieve_trace t, const uint64_t* rep_cycles, sieve_prediction* out) {
  return predict_impl(s, t, 1, rep_cycles, out);
}

extern "C" int sieve_predict_multi(sieve_strata s, sieve_trace t, uint32_t M, const uint64_t* rep_cycles,
                                   sieve_prediction* out) {
  if (M == 0) return SIEVE_OK;
  if (!rep_cycles) return sv_fail(SIEVE_EINVAL, "rep_cycles [M][n_strata] is required");
  return predict_impl(s, t, M, rep_cycles, out);
}

// ------------------------------------------------------------------------------------------
// sieve_load_csv: the profiler's CSV parsed and interned on the GPU
// ------------------------------------------------------------------------------------------
extern "C" int sieve_load_csv(sieve_ctx ctx, const char* data, uint64_t bytes, uint32_t mem,
                              const sieve_csv_spec* spec, uint64_t first_id, sieve_trace* out,
                              uint32_t* num_kernels) {
  if (!out) return sv_fail(SIEVE_EINVAL, "out is NULL");
  *out = nullptr;
  if (!ctx_ok(ctx) || !spec || (bytes && !data)) return sv_fail(SIEVE_EINVAL, "bad argument");
  if (spec->col_kernel < 0 || spec->col_instr < 0) return sv_fail(SIEVE_EINVAL, "kernel and instruction columns are required");
  if (mem & ~1u) return sv_fail(SIEVE_EINVAL, "mem must be SIEVE_MEM_HOST or SIEVE_MEM_DEVICE");
  sieve_ctx c = ctx;
  cudaStream_t S = c->stream;
  SV_CUDA(cudaSetDevice(c->device));
  SV_TRY(arena_reset(c));
  // the bytes on the device (host text: one upload; the names are read from the host text, or,
  // for device-resident text, gathered on the device and only they come back)
  const bool dev_text = (mem & SIEVE_MEM_DEVICE) != 0;
  const unsigned char* dbuf = (const unsigned char*)data;
  const char* hbuf = dev_text ? nullptr : data;
  if (!dev_text) {
    DBuf<unsigned char> db(c);
    SV_TRY(db.alloc(bytes ? bytes : 1));
    if (bytes) SV_CUDA(cudaMemcpyAsync(db.get(), data, bytes, cudaMemcpyHostToDevice, S));
    dbuf = db.get();
  }
  // 1. line ends
  const u64 nt = csv_tiles(bytes);
  DBuf<u32> tiles(c);
  DBuf<char> stemp(c);
  SV_TRY(tiles.alloc(nt + 1));
  SV_TRY(stemp.alloc(scan_u32_temp_bytes(nt + 1)));
  SV_CUDA(cudaMemsetAsync(tiles.get(), 0, (nt + 1) * 4, S));
  launch_csv_count(dbuf, bytes, tiles.get(), stemp.get(), S);
  std::vector<u32> h_nl;
  SV_TRY(d2h(c, h_nl, tiles.get() + nt, 1));
  char last = 0;   // the text's last byte (device-resident text: read with the line count)
  if (bytes && dev_text) SV_TRY(d2h_raw(c, &last, dbuf + bytes - 1, 1));
  SV_TRY(sync(c));
  const u64 nends = h_nl[0];
  DBuf<u64> ends(c);
  SV_TRY(ends.alloc(nends + 1));
  launch_csv_ends(dbuf, bytes, tiles.get(), ends.get(), S);
  const bool trailing = bytes > 0 && (dev_text ? last : hbuf[bytes - 1]) == '\n';
  const u64 nlines = nends + (bytes > 0 && !trailing ? 1 : 0);
  const u64 nrows = nlines > spec->header_lines ? nlines - spec->header_lines : 0;
  if (nrows >= (1ull << 32)) return sv_fail(SIEVE_ERANGE, "more than 2^32 - 1 rows");
  // 2. parse
  DBuf<u64> hash(c), npos(c), errf(c);
  DBuf<u32> row(c);
  SV_TRY(hash.alloc(nrows)); SV_TRY(npos.alloc(2 * nrows)); SV_TRY(errf.alloc(1)); SV_TRY(row.alloc(nrows));
  SV_CUDA(cudaMemsetAsync(errf.get(), 0, 8, S));
  sieve_trace_s* t = new sieve_trace_s();
  t->ctx = c; t->n = nrows; t->first_id = first_id; t->owned = true;
  t->owner = cur_owner(c);
  auto fail = [&](int st) { cudaStreamSynchronize(S); sieve_trace_free(t); return st; };
#define CSV_TRY(e) do { int _s = (e); if (_s != SIEVE_OK) return fail(_s); } while (0)
  void* p;
  int st = SIEVE_OK;
  if ((st = dalloc(c, &p, nrows * 4 + 16)) != SIEVE_OK) return fail(st);
  t->kid = (u32*)p;
  if ((st = dalloc(c, &p, nrows * 8 + 16)) != SIEVE_OK) return fail(st);
  t->x = (u64*)p;
  if (spec->col_cta >= 0) { if ((st = dalloc(c, &p, nrows * 4 + 16)) != SIEVE_OK) return fail(st); t->cta = (u32*)p; }
  if (spec->col_cycles >= 0) { if ((st = dalloc(c, &p, nrows * 8 + 16)) != SIEVE_OK) return fail(st); t->y = (u64*)p; }
  CsvSpec cs{spec->col_kernel, spec->col_instr, spec->col_cta, spec->col_cycles, (unsigned char)spec->delimiter};
  launch_csv_parse(dbuf, bytes, ends.get(), nends, spec->header_lines, nrows, cs, hash.get(), row.get(),
                   npos.get(), t->x, t->cta, t->y, errf.get(), S);
  // 3. intern names: stable sort by hash, distinct heads, ids by first appearance
  std::vector<u64> h_err, h_names;
  std::vector<u32> h_nd;
  u64 nd = 0;
  if (nrows) {
    {
      DBuf<char> tmp(c);
      if ((st = tmp.alloc(radix_sort_temp_bytes(nrows, true))) != SIEVE_OK) return fail(st);
      if ((st = radix_sort(hash.get(), row.get(), nrows, 64, tmp.get(), S)) != SIEVE_OK) return fail(st);
    }
    DBuf<u32> flag(c), seg(c);
    DBuf<char> st2(c);
    CSV_TRY(flag.alloc(nrows)); CSV_TRY(seg.alloc(nrows + 1)); CSV_TRY(st2.alloc(scan_u32_temp_bytes(nrows)));
    launch_csv_heads(hash.get(), nrows, flag.get(), S);
    scan_u32(flag.get(), seg.get(), nrows, st2.get(), seg.get() + nrows, S);
    CSV_TRY(d2h(c, h_nd, seg.get() + nrows, 1));
    CSV_TRY(d2h(c, h_err, errf.get(), 1));
    if ((st = sync(c)) != SIEVE_OK) return fail(st);
    nd = h_nd[0];
    if (h_err[0]) return fail(sv_fail(SIEVE_EINVAL, "malformed CSV row (missing field or non-integer count)"));
    if (nd > SIEVE_MAX_K) return fail(sv_fail(SIEVE_ERANGE, "more than 65536 distinct kernel names"));
    DBuf<u64> fkey(c), names(c);
    DBuf<u32> fval(c), id_of(c);
    CSV_TRY(fkey.alloc(nd)); CSV_TRY(fval.alloc(nd)); CSV_TRY(id_of.alloc(nd)); CSV_TRY(names.alloc(2 * nd));
    launch_csv_firsts(flag.get(), seg.get(), row.get(), nrows, fkey.get(), fval.get(), S);
    {
      DBuf<char> tmp(c);
      if ((st = tmp.alloc(radix_sort_temp_bytes(nd, true, 32))) != SIEVE_OK) return fail(st);
      if ((st = radix_sort(fkey.get(), fval.get(), nd, 32, tmp.get(), S)) != SIEVE_OK) return fail(st);
    }
    launch_csv_ids(fval.get(), nd, id_of.get(), flag.get(), seg.get(), row.get(), nrows, t->kid, S);
    launch_gather_pairs(npos.get(), fkey.get(), nd, names.get(), S);  // first row of each id
    CSV_TRY(d2h(c, h_names, names.get(), 2 * nd));
    if ((st = sync(c)) != SIEVE_OK) return fail(st);
    { cudaError_t ce = cudaGetLastError(); if (ce) return fail(sv_cuda(ce, "csv kernels", __LINE__)); }
  }
  std::vector<unsigned char> h_text;   // device-resident text: the distinct names' bytes only
  std::vector<u64> name_off(nd + 1, 0);
  if (dev_text && nd) {
    for (u64 d = 0; d < nd; d++) name_off[d + 1] = name_off[d] + h_names[2 * d + 1];
    DBuf<u64> d_pos(c), d_off(c);
    DBuf<unsigned char> d_txt(c);
    CSV_TRY(d_pos.alloc(2 * nd)); CSV_TRY(d_off.alloc(nd + 1)); CSV_TRY(d_txt.alloc(name_off[nd] + 1));
    CSV_TRY(h2d(c, d_pos.get(), h_names));
    CSV_TRY(h2d(c, d_off.get(), name_off));
    launch_csv_names(dbuf, d_pos.get(), d_off.get(), nd, d_txt.get(), S);
    CSV_TRY(d2h(c, h_text, d_txt.get(), name_off[nd]));
    if ((st = sync(c)) != SIEVE_OK) return fail(st);
  }
  t->K = nd ? (u32)nd : 1;
  t->names.resize(nd);
  for (u64 d = 0; d < nd; d++) {
    std::string s;
    const char* q = dev_text ? (const char*)h_text.data() + name_off[d] : hbuf + h_names[2 * d];
    for (u64 i = 0; i < h_names[2 * d + 1]; i++) if (q[i] != '"') s.push_back(q[i]);
    t->names[d] = s;
  }
  if (num_kernels) *num_kernels = (uint32_t)nd;
  *out = t;
#undef CSV_TRY
  return SIEVE_OK;
}

// copy a trace's columns back to HOST buffers (each nullable; a column the trace lacks is left
// untouched); *n_local / *num_kernels nullable
extern "C" int sieve_trace_copy(sieve_trace t, uint32_t* kernel_id, uint64_t* instr, uint32_t* cta,
                                uint64_t* cycles, uint64_t* n_local, uint32_t* num_kernels) {
  if (!trace_ok(t)) return sv_fail(SIEVE_EINVAL, "bad trace handle");
  sieve_ctx c = t->ctx;
  SV_CUDA(cudaSetDevice(c->device));
  if (n_local) *n_local = t->n;
  if (num_kernels) *num_kernels = t->K;
  auto cp = [&](void* dst, const void* src, size_t bytes) -> int {
    if (dst && src && bytes) SV_CUDA(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDeviceToHost, c->stream));
    return SIEVE_OK;
  };
  SV_TRY(cp(kernel_id, t->kid, t->n * 4));
  SV_TRY(cp(instr, t->x, t->n * 8));
  SV_TRY(cp(cta, t->cta, t->n * 4));
  SV_TRY(cp(cycles, t->y, t->n * 8));
  SV_CUDA(cudaStreamSynchronize(c->stream));
  return SIEVE_OK;
}

// kernel names of a CSV-loaded trace, in id order, each terminated by '\n'; *needed = bytes
extern "C" int sieve_trace_kernel_names(sieve_trace t, char* buf, uint64_t cap, uint64_t* needed) {
  if (!trace_ok(t)) return sv_fail(SIEVE_EINVAL, "bad trace handle");
  u64 need = 0;
  for (auto& s : t->names) need += s.size() + 1;
  if (needed) *needed = need;
  if (buf) {
    u64 o = 0;
    for (auto& s : t->names) {
      if (o + s.size() + 1 > cap) break;
      memcpy(buf + o, s.data(), s.size());
      o += s.size();
      buf[o++] = '\n';
    }
  }
  return SIEVE_OK;
}
