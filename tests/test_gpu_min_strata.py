"""NEXT-3: exact min-strata DP on the GPU (sieve_min_strata) against the CPU
oracle (oracle_min_strata, reading A28).  Counts and the canonical
optimal cuts must be bit-exact."""
import random
import time

import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu


def _gpu(tr, K, theta=(2, 5), cap=0):
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    ctx = sieve.Ctx(device=0)
    t = sieve.load_trace(ctx, tr["kid"], tr["x"], num_kernels=K)
    return sieve.min_strata(t, theta, cap)


@pytest.mark.parametrize("name,n,cap", [("C1", None, 4000), ("C2", 200000, 3000)])
@pytest.mark.parametrize("theta", [(1, 10), (2, 5), (1, 1)])
def test_matches_oracle(name, n, cap, theta):
    tr = gen.make_trace(name, 0, n)
    K = tr["K"]
    gc, gcuts = _gpu(tr, K, theta, cap)
    oc, ocuts = oracle.min_strata(tr["kid"], tr["x"], K, theta, max_distinct=cap)
    assert gc.tolist() == oc.tolist()
    assert gcuts == ocuts


@pytest.mark.parametrize("seed", range(4))
def test_random_micro_traces(seed):
    rng = np.random.default_rng(0x3D0 + seed)
    K = 30
    n = 4000
    kid = rng.integers(0, K, n).astype(np.uint32)
    x = np.zeros(n, np.uint64)
    for k in range(K):
        rows = kid == k
        kind = k % 3
        if kind == 0:
            x[rows] = rng.integers(1, 50, rows.sum())
        elif kind == 1:
            x[rows] = (rng.pareto(1.2, rows.sum()) * 1e5 + 1).astype(np.uint64)
        else:
            x[rows] = rng.choice([100, 101, 5000, 5003, 80000], rows.sum())
    tr = {"kid": kid, "x": x}
    for theta in [(1, 20), (2, 5), (3, 7)]:
        gc, gcuts = _gpu(tr, K, theta)
        oc, ocuts = oracle.min_strata(kid, x, K, theta, max_distinct=16384)
        assert gc.tolist() == oc.tolist() and gcuts == ocuts


def test_edges_and_errors():
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    ctx = sieve.Ctx(device=0)
    # powers of ten: every value alone; a kernel without invocations; Tier-1
    kid = np.array([0] * 6 + [2] * 3, np.uint32)
    x = np.array([10**i for i in range(1, 7)] + [9, 9, 9], np.uint64)
    t = sieve.load_trace(ctx, kid, x, num_kernels=3)
    counts, cuts = sieve.min_strata(t, (1, 10))
    assert counts.tolist() == [6, 0, 1] and cuts == [[10**i for i in range(2, 7)], [], []]
    # cuts buffer too small -> ERANGE; skipped kernels -> UINT32_MAX
    cbuf = np.zeros(2, np.uint64)
    cnt = np.zeros(3, np.uint32)
    import ctypes
    nc = ctypes.c_uint64()
    rc = sieve.sieve._L.sieve_min_strata(t._h, 1, 10, 0, cnt.ctypes.data_as(ctypes.c_void_p),
                                         cbuf.ctypes.data_as(ctypes.c_void_p), 2, ctypes.byref(nc))
    assert rc == sieve.sieve.SIEVE_ERANGE and nc.value == 5
    counts, cuts = sieve.min_strata(t, (1, 10), max_distinct=5)
    assert counts.tolist() == [0xFFFFFFFF, 0, 1] and cuts == [[], [], []]
    # empty trace
    t0 = sieve.load_trace(ctx, np.zeros(0, np.uint32), np.zeros(0, np.uint64), num_kernels=2)
    assert sieve.min_strata(t0)[0].tolist() == [0, 0]


def test_sieve_never_fewer_and_timing():
    """Quality reference for the KDE reading: Sieve's strata count >= the optimum per kernel."""
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    tr = gen.make_trace("C2")
    K = tr["K"]
    ctx = sieve.Ctx(device=0)
    t = sieve.load_trace(ctx, tr["kid"], tr["x"], num_kernels=K, cta=tr["cta"], cycles=tr["y"])
    st = sieve.stratify(t)
    t0 = time.perf_counter()
    counts, _ = sieve.min_strata(t, max_distinct=1 << 20)
    dt = time.perf_counter() - t0
    per = np.bincount(st.table["kernel_id"], minlength=K)
    ok = counts != 0xFFFFFFFF
    assert np.all(per[ok] >= counts[ok])
    print(f"C2: optimum {int(counts[ok].sum())} strata vs Sieve {int(per[ok].sum())}, DP {dt * 1e3:.1f} ms")
