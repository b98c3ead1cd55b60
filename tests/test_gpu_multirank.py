"""The multi-rank path on ONE GPU: R ranks as host threads in an in-process group (the same
exact limb reductions the NCCL path uses), each holding a contiguous slice of the trace.  The
strata must be byte-identical to R = 1 and to the oracle; per-rank stratum ids must
concatenate to the single-rank ids (byte-identical across R)."""
import threading

import numpy as np
import pytest

import gen
from paper_conf_ispass_naderantahanse23_b200.distributed import shard_bounds
from tests.gpu_helpers import assert_tables_equal, run_gpu, run_oracle

pytestmark = pytest.mark.gpu


def _run_group(tr, world, G=1024):
    import torch
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    grp = sieve.Group(world)
    n = len(tr["kid"])
    res = [None] * world
    errs = []

    def rank_main(r):
        try:
            torch.cuda.set_device(0)
            s = torch.cuda.Stream()
            ctx = sieve.Ctx(device=0, stream=s, rank=r, group=grp)
            first, cnt = shard_bounds(n, world, r)
            sl = slice(first, first + cnt)
            trace = sieve.load_trace(ctx, tr["kid"][sl], tr["x"][sl], num_kernels=tr["K"],
                                     cta=tr["cta"][sl], cycles=tr["y"][sl], first_id=first)
            with torch.cuda.stream(s):
                sid = torch.empty(max(cnt, 1), dtype=torch.int32, device="cuda")
            st = sieve.stratify(trace, stratum_of_invocation=sid, grid_points=G)
            pred = sieve.predict(st, trace)
            s.synchronize()
            res[r] = (st.table.copy(), sid[:cnt].cpu().numpy().view(np.uint32), pred)
            del st, trace, ctx
        except Exception as e:  # pragma: no cover - reported below
            errs.append((r, repr(e)))

    th = [threading.Thread(target=rank_main, args=(r,)) for r in range(world)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=600)
    assert not errs, errs
    return res


@pytest.mark.parametrize("name,world", [("C1", 2), ("C2", 2), ("C2", 3), ("C2", 4)])
def test_group_ranks_identical(name, world):
    tr = gen.make_trace(name)
    one = run_gpu(tr)
    o = run_oracle(tr)
    res = _run_group(tr, world)
    for table, _, _ in res:
        assert table.tobytes() == one["table"].tobytes()
    assert_tables_equal(res[0][0], o.strata)
    sid = np.concatenate([r[1] for r in res])
    assert np.array_equal(sid, one["sid"])
    assert np.array_equal(sid, o.sid)
    preds = [r[2] for r in res]
    assert all(p == preds[0] for p in preds)


def test_group_sweep_tree_identical():
    """The theta sweep's refinement tree on a 3-rank group: every rank records the same tree from
    the replicated part records, so each theta's table equals the single-rank sweep's."""
    import torch
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    tr = gen.make_trace("C2", n=300_000)
    thetas = [(2, 5), (1, 10), (1, 1), (3, 10)]
    ctx1 = sieve.Ctx(device=0)
    t1 = sieve.load_trace(ctx1, tr["kid"], tr["x"], num_kernels=tr["K"], cta=tr["cta"], cycles=tr["y"])
    ref = [s.table.copy() for s in sieve.stratify_sweep(t1, thetas)]
    world, n = 3, len(tr["kid"])
    grp = sieve.Group(world)
    res, errs = [None] * world, []

    def rank_main(r):
        try:
            torch.cuda.set_device(0)
            s = torch.cuda.Stream()
            ctx = sieve.Ctx(device=0, stream=s, rank=r, group=grp)
            first, cnt = shard_bounds(n, world, r)
            sl = slice(first, first + cnt)
            trace = sieve.load_trace(ctx, tr["kid"][sl], tr["x"][sl], num_kernels=tr["K"],
                                     cta=tr["cta"][sl], cycles=tr["y"][sl], first_id=first)
            res[r] = [st.table.copy() for st in sieve.stratify_sweep(trace, thetas)]
            s.synchronize()
        except Exception as e:  # pragma: no cover - reported below
            errs.append((r, repr(e)))

    th = [threading.Thread(target=rank_main, args=(r,)) for r in range(world)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=600)
    assert not errs, errs
    for tables in res:
        for a, b in zip(tables, ref):
            assert a.tobytes() == b.tobytes()


def test_group_rank_with_empty_slice():
    tr = gen.make_trace("C1")
    tr = {k: (v[:3] if isinstance(v, np.ndarray) else v) for k, v in tr.items()}
    res = _run_group(tr, 4)   # rank 3 holds no invocation
    o = run_oracle(tr)
    for table, _, _ in res:
        assert_tables_equal(table, o.strata)


def test_nccl_path_single_rank():
    """The NCCL communicator path (dlopen of libnccl, ncclCommInitRank, ncclAllReduce on every
    reduction) with one rank must give exactly the no-communicator result."""
    import torch
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    tr = gen.make_trace("C2")
    one = run_gpu(tr)
    uid = sieve.get_unique_id()
    ctx = sieve.Ctx(device=0, rank=0, world=1, nccl_id=uid)
    trace = sieve.load_trace(ctx, tr["kid"], tr["x"], num_kernels=tr["K"], cta=tr["cta"], cycles=tr["y"])
    sid = torch.empty(len(tr["kid"]), dtype=torch.int32, device="cuda")
    st = sieve.stratify(trace, stratum_of_invocation=sid)
    torch.cuda.synchronize()
    assert st.table.tobytes() == one["table"].tobytes()
    assert np.array_equal(sid.cpu().numpy().view(np.uint32), one["sid"])


@pytest.mark.parametrize("world", [1, 3])
def test_part_slot_overflow_redo(world, monkeypatch):
    """SIEVE_PART_SLOTS=1 leaves one part slot per round, so every round with more parts redoes
    its part moments (and their all-reduce) with the exact count; results unchanged"""
    monkeypatch.setenv("SIEVE_PART_SLOTS", "1")
    tr = gen.make_trace("C2", n=150_000)
    o = run_oracle(tr)
    if world == 1:
        g = run_gpu(tr)
        assert_tables_equal(g["table"], o.strata)
        assert np.array_equal(g["sid"], o.sid)
    else:
        res = _run_group(tr, world)
        for table, _, _ in res:
            assert_tables_equal(table, o.strata)
        assert np.array_equal(np.concatenate([r[1] for r in res]), o.sid)
