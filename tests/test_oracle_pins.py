"""Pins of the CPU oracle against things other than itself (closed forms, libm, scikit-learn,
scipy, hand-built sequences, symmetry).  Each test names the PAPER.md passage (P:NN) or the
DESIGN.md reading (A*) it checks."""
import math
import random
from fractions import Fraction

import numpy as np
import pytest

import oracle
from oracle import brute

TWO40 = 2.0 ** 40   # A10: densities in units of 2^-40 of one kernel's peak


# ---------------------------------------------------------------- O3 tiers
@pytest.mark.parametrize("vals,expect", [
    ([5, 5, 5], 1),                      # identical counts -> Tier-1
    ([4, 6], 2),                         # CoV = 1/5 < 2/5 -> Tier-2
    ([3, 7], 3),                         # CoV = 2/5 exactly -> Tier-3 ("otherwise"; A2)
    ([5, 17, 17, 21], 3),                # CoV = 6/15 = 2/5 exactly -> Tier-3
    ([11, 23, 27, 39], 3),               # CoV = 2/5 exactly (mu 25, sigma 10)
    ([1, 9], 3),                         # CoV = 4/5
    ([2 ** 40, 2 ** 40 + 1] * 3, 2),     # tiny variance that fp64 one-pass loses (A4)
    ([123456789], 1),                    # n = 1
    ([10, 10, 10, 11], 2),
])
def test_tier_closed_forms(vals, expect):
    assert oracle.tier(vals) == expect


def test_tier_boundary_multisets_exact():
    # every multiset of 2..4 values < 40 whose population CoV is exactly 2/5 must be Tier-3,
    # and nudging theta up by 1/1000 must make it Tier-2 (the boundary is exact, A3)
    found = 0
    for a in range(1, 40):
        for b in range(a + 1, 40):
            v = [a, b]
            mu = Fraction(a + b, 2)
            var = (Fraction(a) - mu) ** 2 / 2 + (Fraction(b) - mu) ** 2 / 2
            if var == Fraction(4, 25) * mu * mu:
                found += 1
                assert oracle.tier(v, (2, 5)) == 3
                assert oracle.tier(v, (401, 1000)) == 2
                assert oracle.tier(v, (399, 1000)) == 3
    assert found >= 5


def test_tier_matches_numpy_away_from_boundary():
    rng = np.random.default_rng(1)
    for _ in range(300):
        n = int(rng.integers(2, 50))
        v = rng.integers(1, 10 ** 6, n)
        cov = v.std() / v.mean()          # numpy: population std (ddof=0)
        if abs(cov - 0.4) < 1e-6 or v.min() == v.max():
            continue
        assert oracle.tier([int(a) for a in v]) == (2 if cov < 0.4 else 3)


def test_tier_theta_variants():
    assert oracle.tier([4, 6], (1, 5)) == 3      # CoV = 1/5 exactly at theta = 0.2
    assert oracle.tier([4, 6], (1, 10)) == 3
    assert oracle.tier([4, 6], (1, 1)) == 2


# ---------------------------------------------------------------- det_exp, Q (A10)
def _decimal_exp2_neg(j):
    from decimal import Decimal, getcontext
    getcontext().prec = 60
    return float(Decimal(2) ** (Decimal(-j) / Decimal(256)))


def test_exp2_tables_correctly_rounded():
    # the oracle's table and the CUDA path's table (kde.cu literals) are each pinned to the
    # correctly rounded 2^(-j/256) for j >= 1 and to 1 - 2^-53 for j = 0 (A10); the two sides
    # share no table generator
    import os
    import re
    want = [1.0 - 2.0 ** -53] + [_decimal_exp2_neg(j) for j in range(1, 256)]
    assert oracle.exp2_table() == want
    src = open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                            "paper_conf_ispass_naderantahanse23_b200", "csrc", "kde.cu")).read()
    body = src[src.index("KDE_EXP2_NEG[256]"):]
    body = body[body.index("{") + 1:body.index("}")]
    got = [float.fromhex(h) for h in re.findall(r"0x[0-9a-fA-F.]+p[+-]?\d+", body)]
    assert got == want


def test_q_terms_are_never_ties():
    """A10: P * T_j * 2^(40-m) is never an exact half-integer, so rint needs no tie rule and the
    GPU may round each term into an integer-valued fp64 accumulator (kde.cu kde_acc).  P*S =
    p*s*2^(a+b) (p, s odd) has fraction 1/2 only if a + b = -1.  P < 2 has a <= 0, and
    S = T * 2^(40-m) with tz trailing zero bits in T's significand has b = tz - 13 - m, so a tie
    needs tz >= 12 + m.  Pin: every table entry has fewer than 12."""
    import struct
    for j, v in enumerate(oracle.exp2_table()):
        bits = struct.unpack("<Q", struct.pack("<d", v))[0]
        mant = (bits & ((1 << 52) - 1)) | (1 << 52)
        tz = (mant & -mant).bit_length() - 1
        assert tz < 12, (j, tz)
    # and directly: random terms of every table entry are never exact half-integers, while the
    # exact power of two T = 1 would produce ties (the reason for 1 - 2^-53)
    rng = random.Random(11)
    ties_with_one = 0
    for _ in range(20000):
        p = 1.0 + rng.randint(-2 ** 40, 2 ** 40) * 2.0 ** -52
        p = math.ldexp(math.floor(math.ldexp(p, 41)), -41) if rng.random() < 0.5 else p
        m = rng.randint(0, 41)
        for T in (oracle.exp2_table()[rng.randrange(256)],):
            v = Fraction(p) * Fraction(T) * Fraction(2) ** (40 - m)
            assert v - math.floor(v) != Fraction(1, 2)
        w = Fraction(p) * Fraction(2) ** (40 - m)
        ties_with_one += (w - math.floor(w) == Fraction(1, 2))
    assert ties_with_one > 0


def test_det_exp_relative_accuracy():
    # degree-3 Taylor on |r| <= ln2/512 plus the one-fma reduction: relative error < 2^-42
    from decimal import Decimal, getcontext
    getcontext().prec = 40
    rng = random.Random(7)
    ts = [0.0, 1e-300, 0.5, 1.0, math.log(2), 28.4, 28.5] + [rng.uniform(0, 28.5) for _ in range(20000)]
    for t in ts:
        e = Decimal(-t).exp()
        d = Decimal(oracle.det_exp(t))
        assert abs(d - e) <= e * Decimal(2) ** -42, (t, d, e)


def test_q_close_to_exact_exponential():
    # Q(t) is within 1 unit (of 2^-40) of e^{-t} 2^40 over the whole window
    from decimal import Decimal, getcontext
    getcontext().prec = 50
    rng = random.Random(9)
    worst = 0
    for t in [0.0, 1e-9, 0.3, 1.0, 5.0, 20.0, 28.4] + [rng.uniform(0, 28.6) for _ in range(5000)]:
        exact = (Decimal(-t).exp() * Decimal(2) ** 40)
        err = abs(Decimal(oracle.q_of_t(t)) - exact)
        worst = max(worst, err)
        assert err <= 1, t
    assert worst > Decimal("0.4")   # the rounding is really to integers at 2^-40


def test_q_matches_exact_fma_emulation():
    # brute.q_of_t emulates fma and the single final rounding with exact rationals; any
    # dropped / added rounding step in the oracle differs somewhere
    rng = random.Random(11)
    for _ in range(2000):
        t = rng.uniform(0, 28.6)
        assert oracle.q_of_t(t) == brute.q_of_t(t)
        assert oracle.det_exp(t) == brute.det_exp(t)


def test_q_cutoff_and_peak():
    assert oracle.q_of_t(0.0) == 2 ** 40
    assert oracle.q_of_t(1.0) == round(math.exp(-1.0) * TWO40)
    # k = rint(t 256 log2 e) > 10526 <=> t > 28.5014 -> 0; e^-28.5014 2^40 = 0.46 rounds to 0
    # anyway, so the cutoff drops nothing the rounding would keep
    assert oracle.q_of_t(28.5) == 0 and oracle.q_of_t(28.6) == 0 and oracle.q_of_t(1e300) == 0
    assert math.exp(-28.5) * TWO40 < 0.5
    assert oracle.q_of_t(27.0) == round(math.exp(-27.0) * TWO40)     # 2.06 -> 2
    assert oracle.q_of_t(28.0) == round(math.exp(-28.0) * TWO40)     # 0.76 -> 1


# ---------------------------------------------------------------- bandwidth ([36]; A8)
def test_bandwidth_scott_normal_reference():
    rng = np.random.default_rng(3)
    for _ in range(50):
        v = rng.integers(1, 10 ** 9, int(rng.integers(2, 3000)))
        h = oracle.bandwidth([int(a) for a in v])
        ref = 1.06 * v.std() * len(v) ** -0.2          # population sigma, Scott's 1.06 n^-1/5
        assert abs(h - ref) <= ref * 2.0 ** -15
        m, e = math.frexp(h)                             # 16 significant bits
        assert (m * 2 ** 16) == int(m * 2 ** 16)


def test_bandwidth_matches_brute():
    rng = random.Random(5)
    for _ in range(100):
        v = [rng.randrange(1, 1 << 44) for _ in range(rng.randrange(2, 40))]
        if min(v) == max(v):
            continue
        assert oracle.bandwidth(v) == brute.bandwidth(v, 1.06)


# ---------------------------------------------------------------- grid (A9)
def test_grid_endpoints_exact():
    for lo, hi, G in [(1, 2, 3), (100, 1000, 1024), (12345, (1 << 44) - 1, 1024), (7, 8, 1000)]:
        assert oracle.grid_point(lo, hi, 0, G) == float(lo)
        assert oracle.grid_point(lo, hi, G - 1, G) == float(hi)


# ---------------------------------------------------------------- KDE ([8] P:317)
def _direct_gauss_sum(vals, grid, h):
    z = (grid[:, None] - vals[None, :].astype(np.float64)) / h
    return np.exp(-0.5 * z * z).sum(axis=1)


def test_kde_against_sklearn_and_scipy():
    from scipy.stats import gaussian_kde
    from sklearn.neighbors import KernelDensity
    rng = np.random.default_rng(12)
    vals = np.concatenate([rng.normal(10_000, 300, 400), rng.normal(14_000, 500, 600)])
    vals = np.clip(np.round(vals), 1, None).astype(np.uint64)
    lo, hi, G = int(vals.min()), int(vals.max()), 256
    h = oracle.bandwidth([int(v) for v in vals])
    D = np.array([float(d) for d in oracle.kde(vals, lo, hi, h, G)]) / TWO40
    grid = np.array([oracle.grid_point(lo, hi, j, G) for j in range(G)])
    n = len(vals)
    kd = KernelDensity(kernel="gaussian", bandwidth=h).fit(vals.astype(np.float64)[:, None])
    sk = np.exp(kd.score_samples(grid[:, None])) * n * h * math.sqrt(2 * math.pi)
    assert np.max(np.abs(D - sk)) <= 1e-12 * sk.max() + 1e-9
    sig1 = vals.astype(np.float64).std(ddof=1)
    sp = gaussian_kde(vals.astype(np.float64), bw_method=h / sig1)(grid) * n * h * math.sqrt(2 * math.pi)
    assert np.max(np.abs(D - sp)) <= 1e-9 * sp.max()
    direct = _direct_gauss_sum(vals, grid, h)
    assert np.max(np.abs(D - direct)) <= 1e-12 * direct.max() + 1e-9


def test_kde_matches_brute_bit_exact():
    rng = random.Random(21)
    vals = [rng.choice([1000, 5000]) + rng.randrange(-50, 50) for _ in range(40)]
    lo, hi, G = min(vals), max(vals), 32
    h = brute.bandwidth(vals, 1.06)
    assert oracle.kde(np.array(vals, np.uint64), lo, hi, h, G) == brute.kde(vals, lo, hi, h, G)


# ---------------------------------------------------------------- valleys (A11)
def test_valleys_hand_built():
    s = 10
    big = 1 << 20
    # zero plateau between two peaks -> one cut at the plateau midpoint
    D = [big, big // 2, 0, 0, 0, 0, 0, big // 2, big]
    assert oracle.valleys(D, s) == [4]
    # ripple below delta -> no cut
    D = [big, big - 3, big - 1, big - 2, big]
    assert oracle.valleys(D, s) == []
    # monotone -> no cut; edges are never valleys
    assert oracle.valleys(list(range(100, 0, -1)), 0) == []
    assert oracle.valleys(list(range(1, 101)), 0) == []
    # k separated peaks -> k-1 cuts
    peak = [0, 50, 100, 50, 0]
    D = peak * 4
    assert oracle.valleys(D, 3) == [4, 9, 14]
    # the minimum's run: the first run of the minimum value wins
    D = [100, 10, 10, 10, 20, 10, 100]
    assert oracle.valleys(D, 2) == [2]
    # agree with the brute force on random sequences
    rng = random.Random(3)
    for _ in range(500):
        D = [rng.randrange(0, 1 << rng.randrange(1, 60)) for _ in range(rng.randrange(3, 64))]
        sh = rng.randrange(0, 12)
        assert oracle.valleys(D, sh) == brute.valley_cuts(D, sh)


# ---------------------------------------------------------------- symmetry pins (O5)
def test_two_point_masses_split_at_midpoint():
    a, b, m = 1000, 10_000, 500
    x = np.array([a] * m + [b] * m, np.uint64)
    kid = np.zeros(2 * m, np.uint32)
    r = oracle.stratify(kid, x, 1, keep_debug=True)
    assert len(r.strata) == 2
    assert list(r.strata["lo"]) == [a, b] and list(r.strata["hi"]) == [a, b]
    seg = r.segments()[0]
    assert seg["split_kind"] == 1 and seg["n_cuts"] == 1
    spacing = (b - a) / 1023
    assert abs(int(seg["cuts"][0]) - math.ceil((a + b) / 2)) <= spacing + 1


def test_bimodal_mixture_one_cut_near_midpoint():
    rng = np.random.default_rng(4)
    mu1, mu2, s = 100_000, 300_000, 4_000       # separation >> 2h (bimodal, textbook)
    x = np.concatenate([rng.normal(mu1, s, 3000), rng.normal(mu2, s, 3000)]).round().astype(np.uint64)
    r = oracle.stratify(np.zeros(len(x), np.uint32), x, 1, keep_debug=True)
    seg = r.segments()[0]
    assert seg["n_cuts"] == 1 and seg["split_kind"] == 1
    assert abs(int(seg["cuts"][0]) - 200_000) < 10_000
    assert len(r.strata) == 2
