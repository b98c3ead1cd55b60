"""The shared input generator: counter-based (slices are order-free) and shaped as stated."""
import numpy as np

import gen


def test_slices_are_consistent():
    g = gen.Generator(gen.get_config("C2"))
    full = g.fill(0, 20_000)
    a = g.fill(0, 7_777)
    b = g.fill(7_777, 20_000 - 7_777)
    for k in ("kid", "x", "cta", "y"):
        assert np.array_equal(full[k], np.concatenate([a[k], b[k]]))


def test_ranges_and_shape():
    tr = gen.make_trace("C1")
    assert tr["x"].min() >= 1 and tr["x"].max() < (1 << 44)
    assert set(np.unique(tr["cta"]).tolist()) <= {64, 128, 256, 512, 1024}
    assert tr["kid"].max() < 20
    g = gen.Generator(gen.get_config("C1"))
    assert sorted(g.kernel_class(k) for k in range(20)) == [1] * 8 + [2] * 6 + [3] * 6


def test_homogeneous_cycles():
    tr = gen.make_trace("C1", homogeneous=1)
    g = gen.Generator(gen.get_config("C1", homogeneous=1))
    ratio = tr["y"] // tr["x"]
    assert np.all(ratio * tr["x"] == tr["y"])
