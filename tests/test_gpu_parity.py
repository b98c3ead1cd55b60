"""GPU parity: the CUDA path (through the C-ABI) against the CPU oracle on identical seeded
inputs.  Integer outputs bit-exact (tiers, strata, per-invocation stratum ids, representatives,
weights, fixed-point densities, cut thresholds); bandwidths bitwise; predictions within 1e-9
relative (north_star tolerance)."""
import random

import numpy as np
import pytest

import gen
from tests.gpu_helpers import (assert_predictions_close, assert_segments_equal,
                               assert_tables_equal, run_gpu, run_oracle)

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


@pytest.mark.parametrize("name", ["C1", "C2"])
def test_config_parity_full(name):
    tr = gen.make_trace(name)
    g = run_gpu(tr, keep_debug=True)
    o = run_oracle(tr, keep_debug=True)
    assert_tables_equal(g["table"], o.strata)
    assert np.array_equal(g["sid"], o.sid)
    assert g["rounds"] == o.rounds
    assert_segments_equal(g["segments"], o.segments())
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    assert_predictions_close(sieve.predict(g["strata"], g["trace"]), o.predict())


def test_c3_parity():
    tr = gen.make_trace("C3")
    g = run_gpu(tr)
    o = run_oracle(tr)
    assert_tables_equal(g["table"], o.strata)
    assert np.array_equal(g["sid"], o.sid)
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    assert_predictions_close(sieve.predict(g["strata"], g["trace"]), o.predict())


@pytest.mark.parametrize("G,ovh", [(3, None), (64, None), (1000, None), (4096, None), (3, "0"), (21, "0"),
                                   (50, "0"), (1000, "0"), (10000, "0")])
def test_grid_sizes(G, ovh, monkeypatch):
    """grid sizes from 3 to 10000, with the default KDE tile plans and with the finest staircase
    forced (ovh "0"): tiles with fewer than 32 live grid points, partial 8-lane groups, and the
    radix cell path (G > 8192)"""
    if ovh is not None:
        monkeypatch.setenv("SIEVE_KDE_OVH", ovh)
    tr = gen.make_trace("C2", n=120_000)
    g = run_gpu(tr, G=G, keep_debug=True)
    o = run_oracle(tr, G=G, keep_debug=True)
    assert_tables_equal(g["table"], o.strata)
    assert np.array_equal(g["sid"], o.sid)
    assert_segments_equal(g["segments"], o.segments())


@pytest.mark.parametrize("group", ["1", "2", "5"])
def test_cell_walk_in_groups(group, monkeypatch):
    """Segments of many value chunks run the cell grouping's per-cell walk in groups of chunks
    (per-group counts, their prefix per segment, then the offsets inside each group); the test
    hook SIEVE_WALK_GROUP forces tiny groups on a C3 slice, whose densities, cuts and strata must
    equal the oracle's."""
    monkeypatch.setenv("SIEVE_WALK_GROUP", group)
    tr = gen.make_trace("C3", n=300_000)
    g = run_gpu(tr, keep_debug=True)
    o = run_oracle(tr, keep_debug=True)
    assert_tables_equal(g["table"], o.strata)
    assert np.array_equal(g["sid"], o.sid)
    assert_segments_equal(g["segments"], o.segments())


@pytest.mark.parametrize("G,radix", [(1024, True), (10000, False)])
def test_cell_radix_path(G, radix, monkeypatch):
    """the onesweep cell-key path (forced by SIEVE_CELL_RADIX, and taken for G > GROUP_MAXG) gives
    the same densities, cuts and strata as the grouped default"""
    if radix:
        monkeypatch.setenv("SIEVE_CELL_RADIX", "1")
    tr = gen.make_trace("C2", n=150_000)
    g = run_gpu(tr, G=G, keep_debug=True)
    o = run_oracle(tr, G=G, keep_debug=True)
    assert_tables_equal(g["table"], o.strata)
    assert np.array_equal(g["sid"], o.sid)
    assert_segments_equal(g["segments"], o.segments())


@pytest.mark.parametrize("G,step", [(1024, 997), (64, 15_999), (1000, 1)])
def test_values_on_grid_boundaries(G, step):
    """a Tier-3 kernel whose values sit on both sides of every round-1 grid point (ceil(g_j) and
    ceil(g_j) - 1, A9 evaluated with IEEE doubles as in the oracle): every cell decision of the
    grouping is a boundary case (the fast path must defer to the exact search), and step = 1
    makes the grid finer than the integers (fast path disabled)"""
    import math
    lo = 1
    hi = lo + (G - 1) * step + 3
    g = [float(lo) + float((hi - lo) * j) / float(G - 1) for j in range(G)]
    vals = sorted({v for j in range(G) for v in (math.ceil(g[j]), math.ceil(g[j]) - 1) if lo <= v <= hi} | {lo, hi})
    rng = np.random.default_rng(G)
    x = np.array(vals * 3, np.uint64)
    kid = np.zeros(len(x), np.uint32)
    filler = np.full(500, 777, np.uint64)  # a Tier-1 kernel
    tr = {"kid": np.concatenate([kid, np.ones(500, np.uint32)]), "x": np.concatenate([x, filler]), "K": 2}
    perm = rng.permutation(len(tr["kid"]))
    tr["kid"], tr["x"] = tr["kid"][perm], tr["x"][perm]
    tr["cta"] = rng.choice(np.array([64, 128], np.uint32), len(perm))
    tr["y"] = (tr["x"] * np.uint64(3)).astype(np.uint64)
    o = run_oracle(tr, G=G, keep_debug=True)
    assert int(o.strata["tier"][0]) == 3
    g_run = run_gpu(tr, G=G, keep_debug=True)
    assert_tables_equal(g_run["table"], o.strata)
    assert np.array_equal(g_run["sid"], o.sid)
    assert_segments_equal(g_run["segments"], o.segments())


@pytest.mark.parametrize("theta", [(1, 10), (1, 2), (1, 1), (3, 7)])
def test_theta_values(theta):
    tr = gen.make_trace("C2", n=100_000)
    g = run_gpu(tr, theta=theta)
    o = run_oracle(tr, theta=theta)
    assert_tables_equal(g["table"], o.strata)
    assert np.array_equal(g["sid"], o.sid)


def test_device_columns_and_nullable_columns():
    tr = gen.make_trace("C1")
    o = run_oracle(tr, cta=False, cycles=False)
    g = run_gpu(tr, cta=False, cycles=False, device_cols=True)
    assert_tables_equal(g["table"], o.strata)
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    with pytest.raises(sieve.SieveError) as e:
        sieve.predict(g["strata"], g["trace"])
    assert e.value.code == -6
    rc = np.arange(1, len(g["table"]) + 1, dtype=np.uint64) * 1000
    assert_predictions_close(sieve.predict(g["strata"], g["trace"], rc), o.predict(rc))


def _micro(seed):
    rng = random.Random(seed)
    n = rng.randrange(1, 3000)
    K = rng.randrange(1, 40)
    kid = np.array([rng.randrange(K) for _ in range(n)], np.uint32)
    modes = {k: [rng.randrange(1, 1 << rng.choice([8, 20, 43])) for _ in range(rng.randrange(1, 5))]
             for k in range(K)}
    x = []
    for k in kid:
        m = rng.choice(modes[int(k)])
        x.append(max(1, min((1 << 44) - 1, m + rng.randrange(-(m // 10) - 1, m // 10 + 2))))
    return {"kid": kid, "x": np.array(x, np.uint64),
            "cta": np.array([rng.choice([32, 64, 1024, 7]) for _ in range(n)], np.uint32),
            "y": np.array([rng.randrange(0, 1 << 40) for _ in range(n)], np.uint64), "K": K}


@pytest.mark.parametrize("seed", range(12))
def test_random_micro_traces(seed):
    tr = _micro(seed)
    G = [3, 17, 128, 1024][seed % 4]
    g = run_gpu(tr, G=G, keep_debug=True)
    o = run_oracle(tr, G=G, keep_debug=True)
    assert_tables_equal(g["table"], o.strata)
    assert np.array_equal(g["sid"], o.sid)
    assert_segments_equal(g["segments"], o.segments())


def test_edge_cases():
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    # empty trace
    tr = {"kid": np.zeros(0, np.uint32), "x": np.zeros(0, np.uint64), "cta": np.zeros(0, np.uint32),
          "y": np.zeros(0, np.uint64), "K": 5}
    g = run_gpu(tr, with_sid=False)
    assert len(g["table"]) == 0
    # single invocation, single kernel
    tr = {"kid": np.zeros(1, np.uint32), "x": np.array([(1 << 44) - 1], np.uint64),
          "cta": np.array([128], np.uint32), "y": np.array([5], np.uint64), "K": 1}
    assert_tables_equal(run_gpu(tr)["table"], run_oracle(tr).strata)
    # every kernel invoked once, values at the edges of the range
    n = 5000
    tr = {"kid": np.arange(n, dtype=np.uint32), "x": np.array([1 + (i * 7919) % ((1 << 44) - 1) for i in range(n)], np.uint64),
          "cta": np.full(n, 256, np.uint32), "y": np.arange(1, n + 1, dtype=np.uint64), "K": n}
    assert_tables_equal(run_gpu(tr)["table"], run_oracle(tr).strata)
    # two equal point masses (symmetric density)
    x = np.array([1000] * 400 + [10_000] * 400, np.uint64)
    tr = {"kid": np.zeros(800, np.uint32), "x": x, "cta": np.full(800, 64, np.uint32),
          "y": x * 3, "K": 1}
    assert_tables_equal(run_gpu(tr)["table"], run_oracle(tr).strata)
    # invalid rows are rejected on the device
    bad = dict(tr)
    bad["x"] = x.copy()
    bad["x"][17] = 0
    with pytest.raises(sieve.SieveError) as e:
        run_gpu(bad)
    assert e.value.code == -2
    bad["x"] = x.copy()
    bad["kid"] = np.zeros(800, np.uint32)
    bad["kid"][5] = 3
    with pytest.raises(sieve.SieveError) as e:
        run_gpu(bad)
    assert e.value.code == -1
    # max_rounds exceeded
    xx = np.array([1, 2, 4, 8, 16, 32, 64, 128, 256, 512, 1024, 2048] * 3, np.uint64)
    tr = {"kid": np.zeros(len(xx), np.uint32), "x": xx, "cta": np.zeros(len(xx), np.uint32),
          "y": xx, "K": 1}
    with pytest.raises(sieve.SieveError) as e:
        run_gpu(tr, max_rounds=1)
    assert e.value.code == -7


@pytest.mark.parametrize("G", [3, 5, 1024])
def test_kde_guarded_variant(G):
    # a huge outlier makes grid steps >> h at small G, so the KDE must take its guarded path
    # (u >= 80 sent to the zero entry explicitly); results must not change
    n = 50_000
    x = np.full(n, 1000, np.uint64)
    x[::997] = 1000 + np.arange(len(x[::997]), dtype=np.uint64) * 3
    x[-1] = 10 ** 12
    tr = {"kid": np.zeros(n, np.uint32), "x": x, "cta": np.full(n, 128, np.uint32),
          "y": x * 2, "K": 1}
    g = run_gpu(tr, G=G, keep_debug=True)
    o = run_oracle(tr, G=G, keep_debug=True)
    assert_tables_equal(g["table"], o.strata)
    assert_segments_equal(g["segments"], o.segments())


def test_many_kernels_multiple_smem_passes():
    # K > 2048 makes pass A run several kernel-id ranges
    rng = np.random.default_rng(3)
    n, K = 200_000, 9000
    kid = rng.integers(0, K, n).astype(np.uint32)
    base = rng.integers(1, 1 << 30, K).astype(np.uint64)
    x = base[kid] + rng.integers(0, 3, n).astype(np.uint64) * (base[kid] // 2)
    tr = {"kid": kid, "x": x, "cta": rng.choice([64, 128], n).astype(np.uint32),
          "y": rng.integers(1, 1 << 30, n).astype(np.uint64), "K": K}
    g = run_gpu(tr)
    o = run_oracle(tr)
    assert_tables_equal(g["table"], o.strata)
    assert np.array_equal(g["sid"], o.sid)


def test_homogeneous_prediction_exact():
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    tr = gen.make_trace("C2", homogeneous=1)
    g = run_gpu(tr)
    p = sieve.predict(g["strata"], g["trace"])
    assert p["error"] < 1e-12


@pytest.mark.parametrize("name,n", [("C1", None), ("C2", 200_000)])
def test_kde_in_window_term_count(name, n):
    """The in-window KDE term count (the roofline's work unit, counted per value in the bucket
    pass) equals a brute-force count over the oracle's segments: pairs (grid point j, value x)
    of every segment of every round with rn(g_j - w) <= x <= rn(g_j + w), w = rn(sqrt(57) h)."""
    tr = gen.make_trace(name, n=n) if n else gen.make_trace(name)
    G = 1024
    g = run_gpu(tr, G=G)
    o = run_oracle(tr, G=G, keep_debug=True)
    wc = np.float64(7.54983443527075)
    j = np.arange(G, dtype=np.int64)
    total = 0
    for seg in o.segments():
        k, lo, hi, h = seg["kernel_id"], int(seg["lo"]), int(seg["hi"]), np.float64(seg["bandwidth"])
        xs = tr["x"][(tr["kid"] == k) & (tr["x"] >= lo) & (tr["x"] <= hi)]
        xs = np.sort(xs.astype(np.float64))  # exact: x < 2^44
        gj = np.float64(lo) + ((hi - lo) * j).astype(np.float64) / np.float64(G - 1)
        w = wc * h
        a = np.searchsorted(xs, gj - w, side="left")
        b = np.searchsorted(xs, gj + w, side="right")
        total += int((b - a).sum())
    assert g["terms"] == total


def test_segment_batches_change_nothing(monkeypatch):
    """A round whose open segments exceed one cell sort's key space runs in batches; forcing
    batches of 3 segments (test hook) must reproduce the oracle exactly."""
    tr = gen.make_trace("C2", n=150_000)
    monkeypatch.setenv("SIEVE_SEG_BATCH", "3")
    g = run_gpu(tr, keep_debug=True)
    o = run_oracle(tr, keep_debug=True)
    assert_tables_equal(g["table"], o.strata)
    assert np.array_equal(g["sid"], o.sid)
    assert_segments_equal(g["segments"], o.segments())


@pytest.mark.parametrize("mode", ["1", "2"])
def test_kde_evaluation_modes_identical(monkeypatch, mode):
    """The KDE evaluates a term three ways (kde.cu kde_acc MODE 0: no k clamp on items proven
    |z| < 18.8; 1: clamped; 2: clamped plus the large-u guard).  The test hook forces the
    slower modes on a whole C2-shaped trace; every density, cut and stratum must still equal the
    oracle's (MODE 0 is what the other parity tests exercise)."""
    tr = gen.make_trace("C2", n=200_000)
    monkeypatch.setenv("SIEVE_KDE_FORCE", mode)
    g = run_gpu(tr, keep_debug=True)
    o = run_oracle(tr, keep_debug=True)
    assert_tables_equal(g["table"], o.strata)
    assert np.array_equal(g["sid"], o.sid)
    assert_segments_equal(g["segments"], o.segments())


def test_kde_staircase_plans_identical(monkeypatch):
    """k_kde_tiles splits each tile's values into regions evaluated by 8, 16 or 32 lanes (the
    staircase at the ends of the tile's window) and picks a plan per tile by estimated cost.
    The test hook SIEVE_KDE_OVH forces the finest staircase everywhere (0) or one 32-lane region
    per tile (inf); both, and the default choice, must give every density, cut and stratum of
    the oracle, and the staircase must evaluate fewer (lane, value) pairs, never fewer than the
    in-window terms."""
    tr = gen.make_trace("C3", n=400_000)
    o = run_oracle(tr, keep_debug=True)
    ev = {}
    for ovh in ["0", "inf", None]:
        if ovh is None:
            monkeypatch.delenv("SIEVE_KDE_OVH", raising=False)
        else:
            monkeypatch.setenv("SIEVE_KDE_OVH", ovh)
        g = run_gpu(tr, keep_debug=True)
        assert_tables_equal(g["table"], o.strata)
        assert np.array_equal(g["sid"], o.sid)
        assert_segments_equal(g["segments"], o.segments())
        ev[ovh] = (g["strata"].kde_evaluated, g["terms"])
    assert ev["0"][1] == ev["inf"][1] == ev[None][1]
    assert ev["0"][1] <= ev["0"][0] < ev["inf"][0]
    assert ev["0"][0] <= ev[None][0] <= ev["inf"][0]


@pytest.mark.parametrize("device", [False, True])
def test_16bit_columns(device):
    """SIEVE_KID16 / SIEVE_CTA16: kernel ids and CTA sizes handed over as uint16 (host or device)
    load the same trace as the 32-bit columns"""
    import torch
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    tr = gen.make_trace("C2", n=80_000)
    o = run_oracle(tr)
    kid16, cta16 = tr["kid"].astype(np.uint16), tr["cta"].astype(np.uint16)
    if device:
        kid16 = torch.from_numpy(kid16.view(np.int16)).cuda()
        cta16 = torch.from_numpy(cta16.view(np.int16)).cuda()
        x = torch.from_numpy(tr["x"].view(np.int64)).cuda()
        y = torch.from_numpy(tr["y"].view(np.int64)).cuda()
    else:
        x, y = tr["x"], tr["y"]
    ctx = sieve.Ctx(device=0)
    t = sieve.load_trace(ctx, kid16, x, num_kernels=tr["K"], cta=cta16, cycles=y)
    kid_back, x_back, cta_back, _ = sieve.trace_columns(t)
    assert np.array_equal(kid_back, tr["kid"]) and np.array_equal(cta_back, tr["cta"])
    sid = torch.empty(len(tr["kid"]), dtype=torch.int32, device="cuda")
    st = sieve.stratify(t, stratum_of_invocation=sid)
    torch.cuda.synchronize()
    assert_tables_equal(st.table, o.strata)
    assert np.array_equal(sid.cpu().numpy().view(np.uint32), o.sid)
    with pytest.raises(sieve.SieveError):
        sieve.load_trace(ctx, kid16 if device else torch.from_numpy(tr["kid"].astype(np.int16)).cuda(),
                         x if device else torch.from_numpy(tr["x"].view(np.int64)).cuda(),
                         num_kernels=tr["K"], adopt=True)


@pytest.mark.parametrize("variant", ["slots2", "4", "hash"])
def test_assign_variants(variant, monkeypatch):
    """pass B's (stratum, CTA) statistics: W fixed slots per stratum (default 2, or 4) and the
    hash-table variant give the oracle's representatives; kernel 0 has seven CTA sizes, so its
    stratum overflows the slots into the L2 table"""
    if variant != "slots2":
        monkeypatch.setenv("SIEVE_ASSIGN", variant)
    tr = gen.make_trace("C2", n=150_000)
    rng = np.random.default_rng(7)
    k0 = np.nonzero(tr["kid"] == 0)[0]
    tr["cta"][k0] = rng.choice(np.array([32, 64, 96, 128, 256, 512, 1024], np.uint32), size=len(k0))
    g = run_gpu(tr)
    o = run_oracle(tr)
    assert_tables_equal(g["table"], o.strata)
    assert np.array_equal(g["sid"], o.sid)
