"""Workload for compute-sanitizer (memcheck / racecheck / synccheck): C1 and a 200k-invocation
slice of C2 through sieve_stratify + sieve_predict (keep_debug on, so every KDE segment is read
back; the C2 slice also with pass B's hash and four-slot variants and the KDE's finest and
coarsest tile plans), plus C1 over an in-process
2-rank group (the multi-rank reduction kernels).

    compute-sanitizer --tool racecheck python tools/sanitize_run.py [--no-group]
"""
import os
import sys
import threading

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ispass_naderantahanse23_b200 as sieve  # noqa: E402
from paper_conf_ispass_naderantahanse23_b200.distributed import shard_bounds  # noqa: E402


def one(tr, n=None, G=1024):
    n = len(tr["kid"]) if n is None else n
    ctx = sieve.Ctx(device=0)
    t = sieve.load_trace(ctx, tr["kid"][:n], tr["x"][:n], num_kernels=tr["K"], cta=tr["cta"][:n],
                         cycles=tr["y"][:n])
    sid = torch.empty(n, dtype=torch.int32, device="cuda")
    st = sieve.stratify(t, stratum_of_invocation=sid, grid_points=G, keep_debug=1)
    segs = st.segments(G)
    p = sieve.predict(st, t)
    torch.cuda.synchronize()
    print(f"n={n} strata={len(st.table)} rounds={st.rounds} segments={len(segs)} "
          f"pred={p['predicted_cycles']:.6g}", flush=True)


def group(tr, world=2):
    grp = sieve.Group(world)
    n = len(tr["kid"])
    errs = []

    def rank_main(r):
        try:
            torch.cuda.set_device(0)
            s = torch.cuda.Stream()
            ctx = sieve.Ctx(device=0, stream=s, rank=r, group=grp)
            first, cnt = shard_bounds(n, world, r)
            sl = slice(first, first + cnt)
            t = sieve.load_trace(ctx, tr["kid"][sl], tr["x"][sl], num_kernels=tr["K"],
                                 cta=tr["cta"][sl], cycles=tr["y"][sl], first_id=first)
            st = sieve.stratify(t)
            sieve.predict(st, t)
            s.synchronize()
        except Exception as e:  # reported below
            errs.append((r, repr(e)))

    th = [threading.Thread(target=rank_main, args=(r,)) for r in range(world)]
    for x in th:
        x.start()
    for x in th:
        x.join()
    assert not errs, errs
    print(f"group world={world} ok", flush=True)


def invalid_rows():
    """rows with x = 0 and a kernel id >= K: the call fails after pass A, while the round-1
    grouping queued behind it still runs over the same rows (it must stay in bounds)"""
    tr = gen.make_trace("C2", n=100_000)
    for bad in ("x", "kid"):
        kid, x = tr["kid"].copy(), tr["x"].copy()
        if bad == "x":
            x[::997] = 0
        else:
            kid[::991] = tr["K"] + 5
        ctx = sieve.Ctx(device=0)
        t = sieve.load_trace(ctx, kid, x, num_kernels=tr["K"], cta=tr["cta"], cycles=tr["y"])
        try:
            sieve.stratify(t)
            raise AssertionError("invalid rows accepted")
        except sieve.SieveError as e:
            print(f"invalid {bad}: status {e.code}", flush=True)
        torch.cuda.synchronize()


def other_entry_points():
    """the rest of the C-ABI on C1-sized inputs: theta sweep, tier census, multi-architecture
    prediction, cycle CoV, exact min-strata DP, CSV ingest, and the radix cell path"""
    import os
    tr = gen.make_trace("C2", n=60_000)
    ctx = sieve.Ctx(device=0)
    t = sieve.load_trace(ctx, tr["kid"], tr["x"], num_kernels=tr["K"], cta=tr["cta"], cycles=tr["y"])
    sts = sieve.stratify_sweep(t, [(1, 10), (2, 5), (1, 1)])
    sieve.tier_census(t, [(1, 10), (2, 5)])
    st = sts[1]
    rc = np.stack([st.table["rep_cycles"], st.table["rep_cycles"] * np.uint64(2)])
    sieve.predict_multi(st, t, rc)
    sid = torch.empty(len(tr["kid"]), dtype=torch.int32, device="cuda")
    st2 = sieve.stratify(t, stratum_of_invocation=sid)
    sieve.cycle_cov(st2, t, sid)
    sieve.min_strata(t, theta=(2, 5))
    lines = ["kernel,instr,cta,cycles"] + [f"k{k},{x},{c},{y}" for k, x, c, y in
                                           zip(tr["kid"][:5000], tr["x"][:5000], tr["cta"][:5000], tr["y"][:5000])]
    tc, names = sieve.load_csv(ctx, "\n".join(lines) + "\n", col_kernel=0, col_instr=1, col_cta=2, col_cycles=3)
    sieve.stratify(tc)
    os.environ["SIEVE_CELL_RADIX"] = "1"
    sieve.stratify(t, grid_points=256)
    del os.environ["SIEVE_CELL_RADIX"]
    torch.cuda.synchronize()
    print("other entry points ok", flush=True)


if __name__ == "__main__":
    other_entry_points()
    invalid_rows()
    one(gen.make_trace("C1"))
    one(gen.make_trace("C2"), n=200_000)
    for v in ("hash", "4"):   # pass B's other variants (two slots per stratum is the default)
        os.environ["SIEVE_ASSIGN"] = v
        one(gen.make_trace("C2"), n=200_000)
    os.environ.pop("SIEVE_ASSIGN", None)
    for v in ("0", "inf"):    # the KDE plans: finest staircase everywhere, one region per tile
        os.environ["SIEVE_KDE_OVH"] = v
        one(gen.make_trace("C2"), n=200_000)
    os.environ.pop("SIEVE_KDE_OVH", None)
    if "--no-group" not in sys.argv:
        group(gen.make_trace("C1"))
    print("sanitize workload done")
