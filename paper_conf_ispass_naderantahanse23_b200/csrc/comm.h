// comm.h -- cross-rank reductions on u64 lanes (SUM / MIN / MAX), the only collective the path
// needs: every cross-rank quantity is additive (counts, 32-bit limbs of u128 sums, fixed-point
// densities, per-(stratum, CTA) counts, owner-contributed representative values) or a min /
// max (smallest / largest instruction count, first invocation id).  See DESIGN.md section 6.
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

#include "common.cuh"

// one in-place all-reduce of n u64 lanes
struct ARReq {
  u64* buf;
  size_t n;
  ReduceOp op;
};

struct Comm {
  int rank = 0, world = 1;
  virtual ~Comm() {}
  // in-place all-reduces of several buffers on `s` as ONE collective step (NCCL: one
  // ncclGroupStart/End group, i.e. one fused launch; in-process group: one set of barriers);
  // every rank passes the same sequence of (n, op).  Returns SIEVE_OK or an error status, and
  // never leaves the other ranks of the group waiting (an error is returned after the step).
  virtual int allreduce_group(const ARReq* reqs, int nreq, cudaStream_t s) = 0;
  int allreduce(u64* buf, size_t n, ReduceOp op, cudaStream_t s) {
    ARReq r{buf, n, op};
    return allreduce_group(&r, 1, s);
  }
};

int nccl_unique_id(uint8_t out[128]);
int nccl_comm_create(int rank, int world, const uint8_t id[128], Comm** out);

struct sieve_group_s;
int group_comm_create(sieve_group_s* g, int rank, Comm** out);
