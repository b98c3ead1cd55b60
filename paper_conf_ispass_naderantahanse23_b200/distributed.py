"""Multi-GPU plumbing for the stratification path.

One process per GPU: each rank holds a contiguous, chronological slice of the invocation
stream (first_id = exclusive prefix of the slice sizes).  Every cross-rank quantity is exact
and additive (u64 lanes; u128 as 32-bit limbs) or a min / max, so the library all-reduces them
with NCCL and every rank takes identical decisions.  torch.distributed only carries the NCCL
unique id from rank 0 to the others.
"""
import os


def shard_bounds(n_total, world, rank):
    """(first_id, n_local) of rank's contiguous slice; sizes differ by at most one."""
    base, rem = divmod(n_total, world)
    first = rank * base + min(rank, rem)
    return first, base + (1 if rank < rem else 0)


def env_rank_world():
    return int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")), \
        int(os.environ.get("LOCAL_RANK", "0"))


def broadcast_unique_id(uid_or_none, src=0, group=None):
    """Send rank 0's NCCL unique id (bytes) to every rank over a torch process group."""
    import torch.distributed as dist
    obj = [uid_or_none]
    dist.broadcast_object_list(obj, src=src, group=group)
    return obj[0]


def make_ctx(device=None, stream=None):
    """Ctx for this process: world 1 without torch.distributed, else an NCCL communicator whose
    unique id travels over the already-initialised torch process group."""
    from .sieve import Ctx, get_unique_id
    import torch
    import torch.distributed as dist
    rank, world, local = env_rank_world()
    if dist.is_available() and dist.is_initialized():
        rank, world = dist.get_rank(), dist.get_world_size()
    device = local if device is None else device
    torch.cuda.set_device(device)
    if world == 1:
        return Ctx(device=device, stream=stream)
    uid = get_unique_id() if rank == 0 else None
    uid = broadcast_unique_id(uid)
    return Ctx(device=device, stream=stream, rank=rank, world=world, nccl_id=uid)


def limb_allreduce_u128(values, group=None):
    """Exact cross-rank sum of Python ints < 2^128 with the library's limb encoding over any
    torch process group (gloo on CPU in the tests, the same encoding NCCL carries on GPUs)."""
    import torch
    import torch.distributed as dist
    from .sieve import limbs_to_u128, u128_to_limbs
    lanes = []
    for v in values:
        lanes.extend(u128_to_limbs(int(v)))
    t = torch.tensor([l for l in lanes], dtype=torch.int64)  # limbs < 2^32 fit int64 exactly
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    out = t.tolist()
    return [limbs_to_u128(out[4 * i:4 * i + 4]) for i in range(len(values))]
