"""C5 (the KDE-stress config: 1B invocations, 2,000 kernels, 40% in Tier-3 kernels with 5-20
modes; BASELINE.json configs[4]) at full size on one B200, in bench.py's launch configuration
(device-resident adopted columns, stratum ids written):
  * properties at any size: partition, weights sum to I, (kernel, lo) order, disjoint intervals,
    one stratum per Tier-1/2 kernel and >= 2 per Tier-3 kernel;
  * a seeded sample of kernels (Tier-3 kernels of 65k to 9M invocations, Tier-1/2 kernels)
    bit-exact against the CPU oracle's strata in tests/golden/c5_subset.json, written by
    tools/make_c5_golden.py (which calls only oracle/ and gen/);
  * 2M sampled per-invocation stratum ids consistent with the table."""
import json
import os

import numpy as np
import pytest

import gen

pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "c5_subset.json")
FIELDS = ["kernel_id", "tier", "index_in_kernel", "rep_cta", "lo", "hi", "count", "instr_sum_lo",
          "instr_sum_hi", "rep_id", "rep_instr", "rep_cycles", "split_round"]
CHUNK = 50_000_000


def test_c5_full_size_against_golden():
    import torch
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    with open(GOLDEN) as f:
        gold = json.load(f)
    cfg = gen.get_config("C5")
    assert (gold["n"], gold["K"], gold["seed"]) == (cfg.n, cfg.K, cfg.seed)
    from tools.make_c5_golden import gen_digest
    assert gold["gen_digest"] == gen_digest(), "generator changed: rerun tools/make_c5_golden.py"
    n = cfg.n
    g = gen.Generator(cfg)
    d = {"kid": torch.empty(n, dtype=torch.int32, device="cuda"),
         "x": torch.empty(n, dtype=torch.int64, device="cuda"),
         "cta": torch.empty(n, dtype=torch.int32, device="cuda"),
         "y": torch.empty(n, dtype=torch.int64, device="cuda")}
    x_sum = 0
    for f in range(0, n, CHUNK):
        m = min(CHUNK, n - f)
        tr = g.fill(f, m)
        x_sum += (int((tr["x"] >> np.uint64(32)).sum()) << 32) + int((tr["x"] & np.uint64(0xFFFFFFFF)).sum())
        for k in d:
            v = tr[k].view(np.int64 if tr[k].dtype == np.uint64 else np.int32)
            d[k][f:f + m].copy_(torch.from_numpy(v))
    ctx = sieve.Ctx(device=0)
    trace = sieve.load_trace(ctx, d["kid"], d["x"], num_kernels=cfg.K, cta=d["cta"], cycles=d["y"],
                             adopt=True)
    sid_t = torch.empty(n, dtype=torch.int32, device="cuda")
    st = sieve.stratify(trace, stratum_of_invocation=sid_t)
    torch.cuda.synchronize()
    T = st.table
    # ---- properties at full size
    assert int(T["count"].sum()) == n
    W = sum((int(h) << 64) | int(l) for l, h in zip(T["instr_sum_lo"], T["instr_sum_hi"]))
    assert W == x_sum
    keys = list(zip(T["kernel_id"].tolist(), T["lo"].tolist()))
    assert keys == sorted(keys)
    for k in np.unique(T["kernel_id"]):
        rows = np.nonzero(T["kernel_id"] == k)[0]
        tiers = set(T["tier"][rows].tolist())
        assert len(tiers) == 1
        assert (len(rows) == 1) == (tiers.pop() in (1, 2))
        assert np.all(T["hi"][rows[:-1]] < T["lo"][rows[1:]])
    # ---- the oracle's strata of the sampled kernels, bit-exact
    pick = sorted(int(k) for k in gold["kernels"])
    G = T[np.isin(T["kernel_id"], pick)]
    O = gold["strata"]
    assert len(G) == len(O)
    for f in FIELDS:
        assert G[f].tolist() == [r[f] for r in O], f
    assert [float(v).hex() for v in G["bandwidth"]] == [r["bandwidth"] for r in O]
    assert {int(s) for s in T["tier"][np.isin(T["kernel_id"], pick)]} >= {1, 2, 3}
    # ---- sampled stratum ids
    rng = np.random.default_rng(5)
    pos = torch.from_numpy(rng.integers(0, n, 2_000_000)).cuda()
    sid = sid_t[pos].cpu().numpy().view(np.uint32)
    kid = d["kid"][pos].cpu().numpy().view(np.uint32)
    x = d["x"][pos].cpu().numpy().view(np.uint64)
    assert np.all(T["kernel_id"][sid] == kid)
    assert np.all((T["lo"][sid] <= x) & (x <= T["hi"][sid]))
