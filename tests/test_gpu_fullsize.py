"""Parity at BASELINE.json's full size (C4: 100M invocations, 2,000 kernels) in the launch
configuration bench.py times (device-resident adopted columns, stratum ids written):
  * properties that hold at any size: partition, weights sum to I, ordering / disjointness,
    one stratum per Tier-1/2 kernel, >= 2 per Tier-3 kernel;
  * sampled outputs the oracle computes one by one: the oracle is separable per kernel, so it
    stratifies a sample of kernels (with their global invocation ids) and their strata must be
    bit-identical to the GPU's; a random sample of per-invocation stratum ids is checked
    against the table."""
import numpy as np
import pytest

import gen
from tests.gpu_helpers import EXACT_FIELDS

pytestmark = pytest.mark.gpu


def _exact_sum_u64(a):
    return (int((a >> np.uint64(32)).sum()) << 32) + int((a & np.uint64(0xFFFFFFFF)).sum())


def test_c4_full_size_sampled_parity():
    import torch
    import oracle
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    cfg = gen.get_config("C4")
    tr = gen.Generator(cfg).fill(0, cfg.n)
    n = cfg.n
    ctx = sieve.Ctx(device=0)
    d = {k: torch.from_numpy(tr[k].view(np.int64 if tr[k].dtype == np.uint64 else np.int32)).cuda()
         for k in ("kid", "x", "cta", "y")}
    trace = sieve.load_trace(ctx, d["kid"], d["x"], num_kernels=cfg.K, cta=d["cta"], cycles=d["y"],
                             adopt=True)
    sid_t = torch.empty(n, dtype=torch.int32, device="cuda")
    st = sieve.stratify(trace, stratum_of_invocation=sid_t)
    torch.cuda.synchronize()
    T = st.table
    # ---- properties at full size
    assert int(T["count"].sum()) == n
    W = sum((int(h) << 64) | int(l) for l, h in zip(T["instr_sum_lo"], T["instr_sum_hi"]))
    assert W == _exact_sum_u64(tr["x"])
    keys = list(zip(T["kernel_id"].tolist(), T["lo"].tolist()))
    assert keys == sorted(keys)
    for k in np.unique(T["kernel_id"]):
        rows = np.nonzero(T["kernel_id"] == k)[0]
        tiers = set(T["tier"][rows].tolist())
        assert len(tiers) == 1
        assert (len(rows) == 1) == (tiers.pop() in (1, 2))
        assert np.all(T["hi"][rows[:-1]] < T["lo"][rows[1:]])
    # ---- sampled stratum ids
    rng = np.random.default_rng(0)
    pos = rng.integers(0, n, 2_000_000)
    sid = sid_t[torch.from_numpy(pos).cuda()].cpu().numpy().view(np.uint32)
    assert np.all(T["kernel_id"][sid] == tr["kid"][pos])
    assert np.all((T["lo"][sid] <= tr["x"][pos]) & (tr["x"][pos] <= T["hi"][sid]))
    # ---- sampled kernels through the oracle, bit-exact
    counts = np.bincount(tr["kid"], minlength=cfg.K)
    tier_of = {int(k): int(t) for k, t in zip(T["kernel_id"], T["tier"])}
    pick = []
    for want, lo, hi, m in [(3, 20_000, 250_000, 5), (3, 50, 20_000, 3), (2, 1000, 10 ** 7, 4), (1, 1, 10 ** 8, 4)]:
        cand = [k for k, t in tier_of.items() if t == want and lo <= counts[k] <= hi]
        pick += list(rng.choice(cand, size=min(m, len(cand)), replace=False))
    # the two largest Tier-3 kernels (~600k invocations each: the widest KDE segments of C4)
    t3 = [k for k, t in tier_of.items() if t == 3]
    pick += sorted(t3, key=lambda k: -counts[k])[:2]
    pick = sorted(set(int(k) for k in pick))
    assert len(pick) >= 12
    rows = np.nonzero(np.isin(tr["kid"], pick))[0]
    o = oracle.stratify(tr["kid"][rows], tr["x"][rows], cfg.K, tr["cta"][rows], tr["y"][rows],
                        ids=rows.astype(np.uint64))
    G = T[np.isin(T["kernel_id"], pick)]
    assert len(G) == len(o.strata)
    for f in EXACT_FIELDS:
        assert np.array_equal(G[f], o.strata[f]), f
    assert np.array_equal(G["bandwidth"].view(np.uint64), o.strata["bandwidth"].view(np.uint64))
