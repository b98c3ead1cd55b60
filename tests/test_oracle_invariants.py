"""Oracle invariants and the big-int brute force on micro traces."""
import math
import random
from fractions import Fraction

import numpy as np
import pytest

import gen
import oracle
from oracle import brute


def _cov_below(vals, theta=Fraction(2, 5)):
    return brute.cov_below([int(v) for v in vals], theta)


def check_invariants(tr, r, theta=Fraction(2, 5)):
    kid, x, cta = tr["kid"], tr["x"], tr.get("cta")
    st = r.strata
    n = len(kid)
    assert int(st["count"].sum()) == n                                   # partition
    W = [(int(h) << 64) | int(l) for l, h in zip(st["instr_sum_lo"], st["instr_sum_hi"])]
    assert sum(W) == int(x.astype(object).sum()) == r.total_instr           # weights sum to 1
    # strata ordered by (kid, lo), disjoint value intervals per kernel
    keys = list(zip(st["kernel_id"].tolist(), st["lo"].tolist()))
    assert keys == sorted(keys)
    sid = r.sid
    assert np.all(st["kernel_id"][sid] == kid)                              # never mix kernels
    assert np.all((st["lo"][sid] <= x) & (x <= st["hi"][sid]))
    per_kernel = {}
    for s in range(len(st)):
        per_kernel.setdefault(int(st["kernel_id"][s]), []).append(s)
    for k, ss in per_kernel.items():
        tiers = {int(st["tier"][s]) for s in ss}
        assert len(tiers) == 1
        t = tiers.pop()
        if t in (1, 2):
            assert len(ss) == 1                                             # one stratum
        else:
            assert len(ss) >= 2                                             # Tier-3: >= 2 reps
        for a, b in zip(ss[:-1], ss[1:]):
            assert st["hi"][a] < st["lo"][b]
    order = np.argsort(sid, kind="stable")
    bounds = np.searchsorted(sid[order], np.arange(len(st) + 1))
    for s in range(len(st)):
        mem = order[bounds[s]:bounds[s + 1]]
        vals = x[mem]
        assert len(mem) == st["count"][s]
        if st["tier"][s] == 1:
            assert vals.min() == vals.max()
            assert st["rep_id"][s] == mem.min()                             # first-chronological
        else:
            assert vals.min() == vals.max() or _cov_below(vals, theta)      # CoV < theta
            c = cta[mem] if cta is not None else np.zeros(len(mem), np.uint32)
            vals_c, inv, counts = np.unique(c, return_inverse=True, return_counts=True)
            firsts = np.array([mem[inv == j].min() for j in range(len(vals_c))])
            best = max(range(len(vals_c)), key=lambda j: (counts[j], -firsts[j]))
            assert st["rep_id"][s] == firsts[best]                           # dominant CTA
            assert st["rep_cta"][s] == vals_c[best]
        assert st["rep_instr"][s] == x[st["rep_id"][s]]


@pytest.mark.parametrize("name", ["C1", "C2"])
def test_invariants_on_configs(name):
    tr = gen.make_trace(name)
    r = oracle.stratify(tr["kid"], tr["x"], tr["K"], tr["cta"], tr["y"])
    check_invariants(tr, r)
    tiers = np.bincount(r.strata["tier"], minlength=4)
    assert tiers[1] > 0 and tiers[2] > 0 and tiers[3] > 0


def _micro_trace(rng, n, K, big):
    kid = np.array([rng.randrange(K) for _ in range(n)], np.uint32)
    modes = {k: [rng.randrange(1, 1 << (40 if big else 12)) for _ in range(rng.randrange(1, 4))]
             for k in range(K)}
    x = []
    for k in kid:
        m = rng.choice(modes[int(k)])
        kind = rng.random()
        if kind < 0.3:
            x.append(m)
        else:
            x.append(max(1, m + rng.randrange(-(m // 20) - 1, m // 20 + 2)))
    cta = np.array([rng.choice([64, 128, 256]) for _ in range(n)], np.uint32)
    y = np.array([rng.randrange(1, 1 << 20) for _ in range(n)], np.uint64)
    return {"kid": kid, "x": np.array(x, np.uint64), "cta": cta, "y": y, "K": K}


@pytest.mark.parametrize("seed", range(8))
def test_brute_force_bit_exact(seed):
    rng = random.Random(seed)
    tr = _micro_trace(rng, rng.randrange(20, 160), rng.randrange(1, 5), big=seed % 2 == 1)
    G = 48
    r = oracle.stratify(tr["kid"], tr["x"], tr["K"], tr["cta"], tr["y"], G=G)
    bs, bsid = brute.stratify(tr["kid"], tr["x"], tr["K"], tr["cta"], tr["y"], G=G)
    st = r.strata
    assert len(st) == len(bs)
    for s, b in zip(st, bs):
        assert (int(s["kernel_id"]), int(s["tier"]), int(s["lo"]), int(s["hi"])) == \
            (b["kid"], b["tier"], b["lo"], b["hi"])
        assert int(s["count"]) == b["count"]
        assert (int(s["instr_sum_hi"]) << 64 | int(s["instr_sum_lo"])) == b["W"]
        assert int(s["rep_id"]) == b["rep"] and int(s["rep_cta"]) == b["rep_cta"]
        assert float(s["bandwidth"]) == b["h"] and int(s["split_round"]) == b["rnd"]
    assert list(r.sid) == bsid
    check_invariants(tr, r)
    p = r.predict()
    bp = brute.predict(bs, tr["y"])
    assert p["predicted_cycles"] == bp["predicted_cycles"]               # float128 then round
    assert math.isclose(p["error"], bp["error"], rel_tol=1e-15, abs_tol=1e-300)
    assert math.isclose(p["speedup"], bp["speedup"], rel_tol=1e-15)


def test_brute_force_densities_bit_exact():
    rng = random.Random(99)
    vals = [rng.choice([300, 900, 2500]) + rng.randrange(-20, 20) for _ in range(60)]
    tr = {"kid": np.zeros(60, np.uint32), "x": np.array(vals, np.uint64)}
    G = 40
    r = oracle.stratify(tr["kid"], tr["x"], 1, G=G, keep_debug=True)
    seg = r.segments()[0]
    h = brute.bandwidth(vals, 1.06)
    D = brute.kde(vals, min(vals), max(vals), h, G)
    assert seg["bandwidth"] == h
    assert [(int(a) | int(b) << 64) for a, b in zip(seg["d_lo"], seg["d_hi"])] == D


# ---------------------------------------------------------------- prediction
def test_homogeneous_cycles_predict_exactly():
    tr = gen.make_trace("C2", homogeneous=1)
    r = oracle.stratify(tr["kid"], tr["x"], tr["K"], tr["cta"], tr["y"])
    p = r.predict()
    # y = a_k x within every kernel => every stratum's IPC is exact => C_pred == C_meas
    assert p["error"] < 1e-15
    assert p["predicted_cycles"] == float(r.c_meas)


def test_tier1_prediction_closed_form():
    # one Tier-1 kernel with varying cycles: C_pred = n * y_first
    n = 50
    x = np.full(n, 777, np.uint64)
    y = np.arange(1000, 1000 + n, dtype=np.uint64)[::-1].copy()
    r = oracle.stratify(np.zeros(n, np.uint32), x, 1, None, y)
    assert r.predict()["predicted_cycles"] == float(n * int(y[0]))


def test_single_invocation_strata_predict_exactly():
    rng = np.random.default_rng(5)
    n = 300
    kid = np.arange(n, dtype=np.uint32)                 # each kernel invoked once
    x = rng.integers(1, 1 << 40, n).astype(np.uint64)
    y = rng.integers(1, 1 << 40, n).astype(np.uint64)
    r = oracle.stratify(kid, x, n, None, y)
    assert len(r.strata) == n
    p = r.predict()
    assert p["error"] < 1e-15 and p["speedup"] == 1.0


def test_cpi_arithmetic_mean_form_identical():
    tr = gen.make_trace("C1")
    r = oracle.stratify(tr["kid"], tr["x"], tr["K"], tr["cta"], tr["y"])
    st = r.strata
    W = [Fraction((int(h) << 64) | int(l)) for l, h in zip(st["instr_sum_lo"], st["instr_sum_hi"])]
    I = sum(W)
    cpi = [Fraction(int(y), int(x)) for x, y in zip(st["rep_instr"], st["rep_cycles"])]
    ipc = [1 / c for c in cpi]
    hm_ipc = 1 / sum((w / I) / v for w, v in zip(W, ipc))
    am_cpi = sum((w / I) * c for w, c in zip(W, cpi))
    assert hm_ipc == 1 / am_cpi
    p = r.predict()
    assert math.isclose(p["predicted_cycles"], float(I / hm_ipc), rel_tol=1e-15)
    assert math.isclose(p["predicted_ipc"], float(hm_ipc), rel_tol=1e-15)
    assert math.isclose(p["speedup"], float(r.c_meas) / float(st["rep_cycles"].astype(object).sum()),
                        rel_tol=1e-15)


def test_user_rep_cycles_without_trace_cycles():
    tr = gen.make_trace("C1")
    r = oracle.stratify(tr["kid"], tr["x"], tr["K"], tr["cta"], None)
    with pytest.raises(oracle.OracleError) as e:
        r.predict()
    assert e.value.code == -6
    p = r.predict(np.ones(len(r.strata), np.uint64))
    assert math.isnan(p["error"]) and p["predicted_cycles"] > 0


def test_errors():
    with pytest.raises(oracle.OracleError) as e:
        oracle.stratify(np.zeros(3, np.uint32), np.array([1, 0, 2], np.uint64), 1)
    assert e.value.code == -2                              # x = 0 rejected (A21)
    with pytest.raises(oracle.OracleError) as e:
        oracle.stratify(np.zeros(3, np.uint32), np.array([1, 1 << 44, 2], np.uint64), 1)
    assert e.value.code == -2
    with pytest.raises(oracle.OracleError) as e:
        oracle.stratify(np.array([0, 5], np.uint32), np.array([1, 2], np.uint64), 2)
    assert e.value.code == -1
    with pytest.raises(oracle.OracleError) as e:
        oracle.stratify(np.zeros(2, np.uint32), np.array([1, 2], np.uint64), 1, theta=(0, 5))
    assert e.value.code == -1
    # max_rounds exceeded -> ELIMIT
    x = np.array([1, 2, 4, 8, 16, 32, 64, 128, 256, 512, 1024, 2048] * 3, np.uint64)
    with pytest.raises(oracle.OracleError) as e:
        oracle.stratify(np.zeros(len(x), np.uint32), x, 1, max_rounds=1)
    assert e.value.code == -7


def test_empty_trace():
    r = oracle.stratify(np.zeros(0, np.uint32), np.zeros(0, np.uint64), 4)
    assert len(r.strata) == 0


# ---------------------------------------------------------------- cycle CoV (Fig. 4)
def test_cycle_cov_definition_and_closed_forms():
    tr = gen.make_trace("C1")
    r = oracle.stratify(tr["kid"], tr["x"], tr["K"], tr["cta"], tr["y"])
    cov, wmean = r.cycle_cov(tr["y"])
    st = r.strata
    order = np.argsort(r.sid, kind="stable")
    bounds = np.searchsorted(r.sid[order], np.arange(len(st) + 1))
    W = [(int(h) << 64) | int(l) for l, h in zip(st["instr_sum_lo"], st["instr_sum_hi"])]
    want = []
    for s in range(len(st)):
        ys = [Fraction(int(v)) for v in tr["y"][order[bounds[s]:bounds[s + 1]]]]
        mu = sum(ys) / len(ys)
        var = sum((v - mu) ** 2 for v in ys) / len(ys)     # population (A1 / A25)
        want.append(math.sqrt(float(var)) / float(mu))
    assert np.allclose(cov, want, rtol=1e-14, atol=0)
    assert math.isclose(wmean, sum(w * c for w, c in zip(W, want)) / sum(W), rel_tol=1e-14)
    # closed forms: constant cycles -> 0; members {y, 3y} -> sigma = y, mu = 2y -> 0.5
    kid = np.zeros(4, np.uint32)
    x = np.array([100, 100, 100, 100], np.uint64)
    r2 = oracle.stratify(kid, x, 1, None, np.array([7, 7, 7, 7], np.uint64))
    assert r2.cycle_cov(np.array([7, 7, 7, 7], np.uint64))[0][0] == 0.0
    y = np.array([5, 15, 5, 15], np.uint64)
    assert r2.cycle_cov(y)[0][0] == 0.5
    with pytest.raises(oracle.OracleError):
        r2.cycle_cov(np.array([1, 1, 1, 1 << 48], np.uint64))
