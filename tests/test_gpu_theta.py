"""NEXT-1: theta studies.  sieve_stratify_sweep must equal independent
sieve_stratify / oracle runs for every theta (it shares pass A, and the refinement tree of the
smallest theta, whose frontier gives every larger theta's strata), and sieve_tier_census must
equal the oracle's tiers (Fig. 2 shape)."""
import numpy as np
import pytest

import gen
from tests.gpu_helpers import assert_tables_equal, run_oracle

pytestmark = pytest.mark.gpu

THETAS = [(1, 10), (1, 5), (2, 5), (1, 2), (1, 1)]


def _trace(name, **kw):
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    tr = gen.make_trace(name, **kw)
    ctx = sieve.Ctx(device=0)
    trace = sieve.load_trace(ctx, tr["kid"], tr["x"], num_kernels=tr["K"], cta=tr["cta"], cycles=tr["y"])
    return tr, ctx, trace


@pytest.mark.parametrize("name", ["C1", "C2"])
def test_sweep_equals_oracle_per_theta(name):
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    tr, ctx, trace = _trace(name)
    outs = sieve.stratify_sweep(trace, THETAS)
    assert len(outs) == len(THETAS)
    for th, st in zip(THETAS, outs):
        o = run_oracle(tr, theta=th)
        assert_tables_equal(st.table, o.strata)
        p = sieve.predict(st, trace)
        q = o.predict()
        assert abs(p["predicted_cycles"] - q["predicted_cycles"]) <= 1e-9 * q["predicted_cycles"]


@pytest.mark.parametrize("G", [64, 1024])
def test_sweep_tree_equals_separate_refinements(G, monkeypatch):
    """The sweep refines once, at the smallest theta, and takes each larger theta's strata from
    that refinement tree; with the thetas unsorted and repeated, every table (and the per-theta
    round counts) must equal what a separate refinement per theta gives (SIEVE_SWEEP_SEPARATE),
    and the tree's results must equal separate sieve_stratify calls."""
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    tr, ctx, trace = _trace("C3", n=600_000)
    thetas = [(1, 2), (1, 10), (3, 10), (1, 10), (2, 5), (1, 1), (7, 10), (1, 20)]
    tree = sieve.stratify_sweep(trace, thetas, grid_points=G)
    monkeypatch.setenv("SIEVE_SWEEP_SEPARATE", "1")
    sep = sieve.stratify_sweep(trace, thetas, grid_points=G)
    monkeypatch.delenv("SIEVE_SWEEP_SEPARATE")
    for th, a, b in zip(thetas, tree, sep):
        assert_tables_equal(a.table, b.table)
        assert a.rounds == b.rounds, th
    for th in [(1, 10), (1, 1)]:
        one = sieve.stratify(trace, theta=th, grid_points=G)
        assert_tables_equal(tree[thetas.index(th)].table, one.table)


def test_sweep_degenerate_theta_lists():
    """A sweep of one theta (no tree), of one theta repeated (the tree and its own root), and of
    an empty list."""
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    tr, ctx, trace = _trace("C2", n=200_000)
    one = sieve.stratify(trace, theta=(2, 5))
    for thetas in ([(2, 5)], [(2, 5), (2, 5), (4, 10)]):
        outs = sieve.stratify_sweep(trace, thetas)
        assert len(outs) == len(thetas)
        for st in outs:
            assert_tables_equal(st.table, one.table)
    assert sieve.stratify_sweep(trace, []) == []


def test_census_matches_oracle_tiers():
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    tr, ctx, trace = _trace("C2")
    k, inv, ins = sieve.tier_census(trace, THETAS)
    x = tr["x"].astype(object)
    for i, th in enumerate(THETAS):
        o = run_oracle(tr, theta=th)
        st = o.strata
        for t in (1, 2, 3):
            rows = st["tier"] == t
            assert k[i, t - 1] == len(np.unique(st["kernel_id"][rows]))
            assert inv[i, t - 1] == int(st["count"][rows].sum())
            W = sum((int(h) << 64) | int(l) for l, h in zip(st["instr_sum_lo"][rows], st["instr_sum_hi"][rows]))
            assert ins[i][t - 1] == W
    # monotone in theta: a larger threshold never moves a kernel up a tier
    assert np.all(np.diff(k[:, 2].astype(np.int64)) <= 0)
    assert sum(inv[0]) == len(tr["kid"])


def test_predict_multi_architecture():
    """NEXT-2 (Fig. 9): the same representatives with M cycle vectors."""
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    tr, ctx, trace = _trace("C2")
    st = sieve.stratify(trace)
    o = run_oracle(tr)
    ns = len(st)
    rng = np.random.default_rng(0)
    base = st.table["rep_cycles"].astype(np.uint64)
    rc = np.stack([base, base * 2, rng.integers(1, 1 << 40, ns).astype(np.uint64)])
    preds = sieve.predict_multi(st, trace, rc)
    for m in range(3):
        q = o.predict(rc[m])
        assert abs(preds[m]["predicted_cycles"] - q["predicted_cycles"]) <= 1e-9 * q["predicted_cycles"]
    # doubling every representative's cycles doubles the prediction (relative speedup 2)
    assert abs(preds[1]["predicted_cycles"] / preds[0]["predicted_cycles"] - 2.0) < 1e-12
    single = sieve.predict(st, trace)
    assert preds[0]["predicted_cycles"] == single["predicted_cycles"]


@pytest.mark.parametrize("name", ["C1", "C2", "manyK"])
def test_cycle_cov_matches_oracle(name):
    """Fig. 4 diagnostic: per-stratum cycle CoV bit-identical to the oracle.  manyK:
    9,000 kernels, 8,742 strata: two shared-memory passes of the per-stratum table (4,608 each)."""
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    from tests.gpu_helpers import run_gpu
    tr = gen.make_trace("C2", K=9000, n=800_000) if name == "manyK" else gen.make_trace(name)
    g = run_gpu(tr)
    import torch
    sid = torch.from_numpy(g["sid"].view(np.int32)).cuda()
    cov, w = sieve.cycle_cov(g["strata"], g["trace"], sid)
    o = run_oracle(tr)
    ocov, ow = o.cycle_cov(tr["y"])
    assert np.array_equal(cov, ocov)
    assert abs(w - ow) <= 1e-12 * max(ow, 1e-300)
    assert 0.0 <= w < 0.5     # within-stratum cycle variability is small (0.09 mean)
