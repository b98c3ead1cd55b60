"""Host-side logic of the N > 1 path on CPU with world_size-2 gloo process groups: contiguous
sharding with first_id offsets, the NCCL unique-id broadcast, and the exact u128 limb
all-reduce that every cross-rank sum of the path uses."""
import os
import socket

import pytest
import torch.multiprocessing as mp

from paper_conf_ispass_naderantahanse23_b200.distributed import shard_bounds


def test_shard_bounds_partition():
    for n in [0, 1, 7, 10_000, 100_000_001]:
        for w in [1, 2, 3, 8]:
            got = [shard_bounds(n, w, r) for r in range(w)]
            assert sum(c for _, c in got) == n
            pos = 0
            for f, c in got:
                assert f == pos
                pos += c
            assert max(c for _, c in got) - min(c for _, c in got) <= 1


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_ispass_naderantahanse23_b200.distributed import (broadcast_unique_id,
                                                                          limb_allreduce_u128,
                                                                          shard_bounds)
        import gen
        # unique-id exchange: rank 0's bytes reach everyone
        uid = bytes(range(128)) if rank == 0 else None
        got = broadcast_unique_id(uid)
        # each rank reduces moments of its own slice; the limb all-reduce gives the exact total
        tr = gen.make_trace("C1")
        first, cnt = shard_bounds(len(tr["kid"]), world, rank)
        x = [int(v) for v in tr["x"][first:first + cnt]]
        big = [(1 << 127) // 3 + rank, (1 << 90) * (rank + 1)]
        s1 = sum(x)
        s2 = sum(v * v for v in x)
        red = limb_allreduce_u128([s1, s2] + big)
        q.put((rank, got, red))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_gloo_two_ranks_exact_limb_reduce(world):
    import gen
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    tr = gen.make_trace("C1")
    x = [int(v) for v in tr["x"]]
    want = [sum(x), sum(v * v for v in x), sum((1 << 127) // 3 + r for r in range(world)),
            sum((1 << 90) * (r + 1) for r in range(world))]
    for rank, uid, red in res:
        assert uid == bytes(range(128))
        assert red == want
