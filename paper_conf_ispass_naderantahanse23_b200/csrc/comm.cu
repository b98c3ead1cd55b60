// comm.cu -- the two Comm backends:
//   * NCCL (one process per GPU over NVLink 5 / NVSwitch): ncclAllReduce on ncclUint64 with
//     ncclSum / ncclMin / ncclMax.  libnccl is loaded with dlopen on first use (the copy that
//     PyTorch ships, or $SIEVE_NCCL_LIB), so single-GPU use never needs NCCL.
//   * in-process group (several ranks as host threads on ONE GPU, for parity tests of the
//     multi-rank path where only one GPU exists): each rank publishes its device buffer, a
//     kernel reduces all ranks' buffers into a private temporary, a second barrier guarantees
//     every rank has finished reading before results are copied back.
#include <dlfcn.h>
#include <stdlib.h>
#include <string.h>

#include <condition_variable>
#include <mutex>
#include <string>
#include <vector>

#include "comm.h"

// ------------------------------------------------------------------------------------------
// NCCL through dlopen (types restated from nccl.h: ncclUint64 = 5, ncclSum = 0, ncclMax = 2,
// ncclMin = 3, ncclSuccess = 0, ncclUniqueId = 128 bytes)
// ------------------------------------------------------------------------------------------
typedef struct { char internal[128]; } nccl_uid_t;
typedef void* nccl_comm_t;
typedef int (*fn_get_uid)(nccl_uid_t*);
typedef int (*fn_init_rank)(nccl_comm_t*, int, nccl_uid_t, int);
typedef int (*fn_allreduce)(const void*, void*, size_t, int, int, nccl_comm_t, cudaStream_t);
typedef int (*fn_destroy)(nccl_comm_t);
typedef const char* (*fn_errstr)(int);
typedef int (*fn_group)(void);

static struct {
  void* h = nullptr;
  fn_get_uid get_uid;
  fn_init_rank init_rank;
  fn_allreduce allreduce;
  fn_destroy destroy;
  fn_errstr errstr;
  fn_group group_start, group_end;
} g_nccl;

static int nccl_load() {
  if (g_nccl.h) return SIEVE_OK;
  std::vector<std::string> cands;
  if (const char* e = getenv("SIEVE_NCCL_LIB")) cands.push_back(e);
  cands.push_back("libnccl.so.2");
  cands.push_back("libnccl.so");
  void* h = nullptr;
  for (auto& c : cands) {
    h = dlopen(c.c_str(), RTLD_NOW | RTLD_GLOBAL);
    if (h) break;
  }
  if (!h) return sv_fail(SIEVE_ENCCL, "cannot dlopen libnccl.so.2 (set SIEVE_NCCL_LIB, or import torch first)");
  g_nccl.get_uid = (fn_get_uid)dlsym(h, "ncclGetUniqueId");
  g_nccl.init_rank = (fn_init_rank)dlsym(h, "ncclCommInitRank");
  g_nccl.allreduce = (fn_allreduce)dlsym(h, "ncclAllReduce");
  g_nccl.destroy = (fn_destroy)dlsym(h, "ncclCommDestroy");
  g_nccl.errstr = (fn_errstr)dlsym(h, "ncclGetErrorString");
  g_nccl.group_start = (fn_group)dlsym(h, "ncclGroupStart");
  g_nccl.group_end = (fn_group)dlsym(h, "ncclGroupEnd");
  if (!g_nccl.get_uid || !g_nccl.init_rank || !g_nccl.allreduce || !g_nccl.destroy ||
      !g_nccl.group_start || !g_nccl.group_end)
    return sv_fail(SIEVE_ENCCL, "libnccl is missing required symbols");
  g_nccl.h = h;
  return SIEVE_OK;
}

static int nccl_check(int r, const char* what) {
  if (r == 0) return SIEVE_OK;
  std::string m = std::string(what) + ": " + (g_nccl.errstr ? g_nccl.errstr(r) : "nccl error");
  return sv_fail(SIEVE_ENCCL, m);
}

int nccl_unique_id(uint8_t out[128]) {
  SV_TRY(nccl_load());
  nccl_uid_t id;
  SV_TRY(nccl_check(g_nccl.get_uid(&id), "ncclGetUniqueId"));
  memcpy(out, id.internal, 128);
  return SIEVE_OK;
}

struct NcclComm : Comm {
  nccl_comm_t c = nullptr;
  ~NcclComm() override {
    if (c) g_nccl.destroy(c);
  }
  int allreduce_group(const ARReq* reqs, int nreq, cudaStream_t s) override {
    int live = 0;
    for (int i = 0; i < nreq; i++) live += reqs[i].n != 0;
    if (!live) return SIEVE_OK;
    SV_TRY(nccl_check(g_nccl.group_start(), "ncclGroupStart"));
    int st = SIEVE_OK;
    for (int i = 0; i < nreq && st == SIEVE_OK; i++) {
      if (!reqs[i].n) continue;
      const int nop = reqs[i].op == RED_SUM ? 0 : (reqs[i].op == RED_MAX ? 2 : 3);
      st = nccl_check(g_nccl.allreduce(reqs[i].buf, reqs[i].buf, reqs[i].n, 5 /* ncclUint64 */, nop, c, s),
                      "ncclAllReduce");
    }
    const int ge = nccl_check(g_nccl.group_end(), "ncclGroupEnd");
    return st != SIEVE_OK ? st : ge;
  }
};

int nccl_comm_create(int rank, int world, const uint8_t id[128], Comm** out) {
  SV_TRY(nccl_load());
  NcclComm* nc = new NcclComm();
  nc->rank = rank;
  nc->world = world;
  nccl_uid_t uid;
  memcpy(uid.internal, id, 128);
  int st = nccl_check(g_nccl.init_rank(&nc->c, world, uid, rank), "ncclCommInitRank");
  if (st != SIEVE_OK) { nc->c = nullptr; delete nc; return st; }
  *out = nc;
  return SIEVE_OK;
}

// ------------------------------------------------------------------------------------------
// in-process group
// ------------------------------------------------------------------------------------------
#define GROUP_MAX 16
#define GROUP_MAXREQ 8
struct sieve_group_s {
  int magic = 0x5e6e0001;
  int world = 0;
  std::mutex m;
  std::condition_variable cv;
  int arrived = 0;
  long generation = 0;
  u64* ptrs[GROUP_MAX][GROUP_MAXREQ] = {};
  int err[GROUP_MAX] = {};
  void barrier() {
    std::unique_lock<std::mutex> lk(m);
    long gen = generation;
    if (++arrived == world) {
      arrived = 0;
      generation++;
      cv.notify_all();
    } else {
      cv.wait(lk, [&] { return generation != gen; });
    }
  }
};

struct PtrPack { const u64* p[GROUP_MAX]; };

__global__ void k_group_reduce(PtrPack pk, int world, size_t n, int op, u64* out) {
  pdl_begin();
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    u64 v = pk.p[0][i];
    for (int r = 1; r < world; r++) {
      u64 w = pk.p[r][i];
      v = op == RED_SUM ? v + w : (op == RED_MIN ? (w < v ? w : v) : (w > v ? w : v));
    }
    out[i] = v;
  }
}

// first CUDA failure of a step, kept so the rank still reaches every barrier of the step (a rank
// that returned early would leave the others waiting forever)
#define GC_CUDA(x)                                                   \
  do {                                                               \
    cudaError_t _e = (x);                                            \
    if (_e != cudaSuccess && st == SIEVE_OK) st = sv_cuda(_e, #x, __LINE__); \
  } while (0)

struct GroupComm : Comm {
  sieve_group_s* g = nullptr;
  int allreduce_group(const ARReq* reqs, int nreq, cudaStream_t s) override {
    // every rank must take part even with n == 0 (identical call sequence on all ranks)
    int st = SIEVE_OK;
    if (nreq > GROUP_MAXREQ) return sv_fail(SIEVE_EINVAL, "internal: too many grouped all-reduces");
    GC_CUDA(cudaStreamSynchronize(s));
    for (int i = 0; i < nreq; i++) g->ptrs[rank][i] = reqs[i].buf;
    g->err[rank] = st;
    g->barrier();
    // a rank whose stream failed makes every rank return an error from this step (together)
    bool peer_failed = false;
    for (int r = 0; r < world; r++) peer_failed |= g->err[r] != SIEVE_OK;
    if (peer_failed && st == SIEVE_OK) st = sv_fail(SIEVE_ECUDA, "another rank of the group failed");
    u64* tmp[GROUP_MAXREQ] = {};
    for (int i = 0; i < nreq && st == SIEVE_OK; i++) {
      const size_t n = reqs[i].n;
      if (!n) continue;
      GC_CUDA(cudaMallocAsync((void**)&tmp[i], n * 8, s));
      if (st != SIEVE_OK) break;
      PtrPack pk;
      for (int r = 0; r < world; r++) pk.p[r] = g->ptrs[r][i];
      unsigned blocks = (unsigned)((n + 255) / 256);
      if (blocks > 4096) blocks = 4096;
      SV_LAUNCH(k_group_reduce, blocks, 256, 0, s)(pk, world, n, (int)reqs[i].op, tmp[i]);
      GC_CUDA(cudaGetLastError());
    }
    GC_CUDA(cudaStreamSynchronize(s));
    g->barrier();  // all ranks have read every buffer
    for (int i = 0; i < nreq; i++) {
      if (!tmp[i]) continue;
      if (st == SIEVE_OK) GC_CUDA(cudaMemcpyAsync(reqs[i].buf, tmp[i], reqs[i].n * 8, cudaMemcpyDeviceToDevice, s));
      GC_CUDA(cudaFreeAsync(tmp[i], s));
    }
    GC_CUDA(cudaStreamSynchronize(s));
    g->barrier();  // nobody reuses a published pointer before everyone copied
    return st;
  }
};

int group_comm_create(sieve_group_s* g, int rank, Comm** out) {
  if (!g || g->magic != 0x5e6e0001 || rank < 0 || rank >= g->world)
    return sv_fail(SIEVE_EINVAL, "bad group or rank");
  GroupComm* c = new GroupComm();
  c->g = g;
  c->rank = rank;
  c->world = g->world;
  *out = c;
  return SIEVE_OK;
}

extern "C" int sieve_group_create(int world, sieve_group* out) {
  if (!out || world < 1 || world > GROUP_MAX) return sv_fail(SIEVE_EINVAL, "group world must be in [1, 16]");
  sieve_group_s* g = new sieve_group_s();
  g->world = world;
  *out = g;
  return SIEVE_OK;
}

extern "C" void sieve_group_destroy(sieve_group g) {
  if (g && g->magic == 0x5e6e0001) { g->magic = 0; delete g; }
}
