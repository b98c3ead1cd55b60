"""Pins of the exact min-strata DP oracle (NEXT-3, reading A28; "(1)
minimises the number of strata such that (2) the CoV of each stratum is below theta").

Pinned against exhaustive enumeration of every partition into runs (oracle/brute.py, Fractions),
closed forms, and the invariant that Sieve's own strata (a feasible partition) are never fewer."""
import random
from fractions import Fraction

import numpy as np
import pytest

import gen
import oracle
from oracle import brute

SKIP = 0xFFFFFFFF


@pytest.mark.parametrize("seed", range(6))
def test_dp_equals_exhaustive_enumeration(seed):
    rng = random.Random(0xD9 + seed)
    kid, x, expect = [], [], []
    K = 40
    for k in range(K):
        m = rng.randint(1, 8)
        base = rng.choice([10, 1000, 10**6])
        vals = sorted({rng.randint(base, base * rng.choice([2, 3, 10])) for _ in range(m)})
        mult = [rng.randint(1, 4) for _ in vals]
        for v, c in zip(vals, mult):
            kid += [k] * c
            x += [v] * c
    order = list(range(len(kid)))
    rng.shuffle(order)
    kid = [kid[i] for i in order]
    x = [x[i] for i in order]
    for theta in [(1, 10), (1, 5), (2, 5), (1, 1)]:
        counts, cuts = oracle.min_strata(kid, x, K, theta)
        for k in range(K):
            vals = [x[i] for i in range(len(x)) if kid[i] == k]
            c, cu = brute.min_strata(vals, Fraction(*theta))
            assert counts[k] == c, (k, theta, vals)
            assert cuts[k] == (cu if c > 1 else []), (k, theta, vals)


def test_closed_forms():
    # all equal -> 1; powers of ten with theta = 1/10 -> every value alone; two tight clusters -> 2
    kid = [0] * 5 + [1] * 6 + [2] * 10
    x = [7] * 5 + [10**i for i in range(1, 7)] + [100] * 5 + [1000] * 5
    counts, cuts = oracle.min_strata(kid, x, 3, (1, 10))
    assert counts.tolist() == [1, 6, 2]
    assert cuts == [[], [10**i for i in range(2, 7)], [1000]]
    # CoV exactly theta is not below theta (A2): {3, 7} has CoV 2/5 exactly -> 2 strata
    counts, cuts = oracle.min_strata([0, 0], [3, 7], 1, (2, 5))
    assert counts.tolist() == [2] and cuts == [[7]]
    counts, _ = oracle.min_strata([0, 0], [3, 7], 1, (2001, 5000))
    assert counts.tolist() == [1]
    # a kernel without invocations -> 0
    counts, _ = oracle.min_strata([1], [5], 2)
    assert counts.tolist() == [0, 1]


def test_skip_cap_applies_only_to_non_trivial_kernels():
    kid = [0] * 50 + [1] * 50
    x = list(range(1000, 1050)) + [2**k for k in range(1, 51)]
    counts, cuts = oracle.min_strata(kid, x, 2, (2, 5), max_distinct=10)
    assert counts[0] == 1 and counts[1] == SKIP and cuts == [[], []]


@pytest.mark.parametrize("name,n", [("C1", None), ("C2", 60000)])
def test_sieve_strata_never_fewer_than_optimum(name, n):
    tr = gen.make_trace(name, 0, n)
    K = tr["K"]
    counts, cuts = oracle.min_strata(tr["kid"], tr["x"], K)
    st = oracle.stratify(tr["kid"], tr["x"], K, tr["cta"], tr["y"]).strata
    per = np.bincount(st["kernel_id"], minlength=K)
    present = np.bincount(tr["kid"], minlength=K) > 0
    assert np.all(counts[~present] == 0)
    assert np.all(counts[present] >= 1)
    assert np.all(per[present] >= counts[present])
    # the optimal cuts define runs that each pass the exact test
    for k in range(K):
        if counts[k] < 2:
            continue
        v = np.sort(tr["x"][tr["kid"] == k]).astype(object)
        bounds = [0] + list(cuts[k]) + [1 << 64]
        assert len(cuts[k]) == counts[k] - 1 and cuts[k] == sorted(cuts[k])
        for a, b in zip(bounds[:-1], bounds[1:]):
            part = [int(w) for w in v if a <= w < b]
            assert part and oracle.tier(part) in (1, 2)
