"""Write tests/golden/c5_subset.json: the CPU oracle's strata for a seeded sample of C5's kernels
(the KDE-stress config, 1B invocations: BASELINE.json configs[4]).

Calls only oracle/ and gen/ (the seeded input module): the oracle is separable per kernel, so
each sampled kernel is stratified from its own rows with their global invocation ids (P:93
"first-chronological" needs them).  tests/test_gpu_c5.py compares the GPU's full-size C5 table
against this file.

    python tools/make_c5_golden.py [--jobs 8]
"""
import argparse
import hashlib
import json
import os
import sys
import time
from concurrent.futures import ProcessPoolExecutor

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import gen  # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "c5_subset.json")
FIELDS = ["kernel_id", "tier", "index_in_kernel", "rep_cta", "lo", "hi", "count", "instr_sum_lo",
          "instr_sum_hi", "rep_id", "rep_instr", "rep_cycles", "split_round"]
CHUNK = 50_000_000
SAMPLE_SEED = 0x51E7E0C5
# (intended class, min invocations, max invocations, how many)
BUCKETS = [(3, 20_000, 500_000, 6), (3, 1_000_000, 3_000_000, 2), (3, 5_000_000, 12_000_000, 1),
           (2, 10_000, 10 ** 8, 2), (1, 10_000, 10 ** 8, 2)]


def gen_digest():
    h = hashlib.sha256()
    for f in ("sieve_gen.h", "gen_host.c", "__init__.py"):
        with open(os.path.join(ROOT, "gen", f), "rb") as fh:
            h.update(fh.read())
    return h.hexdigest()[:16]


def collect(cfg, pick):
    g = gen.Generator(cfg)
    rows = {k: [] for k in pick}
    cols = {k: {"x": [], "cta": [], "y": []} for k in pick}
    pick_arr = np.array(sorted(pick), np.uint32)
    for f in range(0, cfg.n, CHUNK):
        tr = g.fill(f, min(CHUNK, cfg.n - f))
        sel = np.nonzero(np.isin(tr["kid"], pick_arr))[0]
        kk = tr["kid"][sel]
        for k in pick:
            s = sel[kk == k]
            rows[k].append(s.astype(np.uint64) + np.uint64(f))
            for c in ("x", "cta", "y"):
                cols[k][c].append(tr[c][s])
    return {k: (np.concatenate(rows[k]), {c: np.concatenate(v) for c, v in cols[k].items()})
            for k in pick}


def run_one(args):
    import oracle
    k, K, ids, c = args
    t = time.time()
    o = oracle.stratify(np.full(len(ids), k, np.uint32), c["x"], K, c["cta"], c["y"], ids=ids)
    st = o.strata
    recs = [{f: int(s[f]) for f in FIELDS} | {"bandwidth": float(s["bandwidth"]).hex()} for s in st]
    return k, recs, o.rounds, time.time() - t


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--jobs", type=int, default=os.cpu_count())
    a = ap.parse_args()
    cfg = gen.get_config("C5")
    g = gen.Generator(cfg)
    counts = np.zeros(cfg.K, np.int64)
    for f in range(0, cfg.n, CHUNK):
        counts += np.bincount(g.fill(f, min(CHUNK, cfg.n - f))["kid"], minlength=cfg.K)
    cls = np.array([g.kernel_class(k) for k in range(cfg.K)])
    rng = np.random.default_rng(SAMPLE_SEED)
    pick = []
    for c, lo, hi, m in BUCKETS:
        cand = [k for k in range(cfg.K) if cls[k] == c and lo <= counts[k] <= hi]
        pick += [int(k) for k in rng.choice(cand, size=min(m, len(cand)), replace=False)]
    pick = sorted(set(pick))
    data = collect(cfg, pick)
    jobs = [(k, cfg.K, data[k][0], data[k][1]) for k in sorted(pick, key=lambda k: -counts[k])]
    out = {"config": "C5", "n": cfg.n, "K": cfg.K, "seed": cfg.seed, "gen_digest": gen_digest(),
           "theta": [2, 5], "grid_points": 1024, "kernels": {}, "strata": []}
    with ProcessPoolExecutor(a.jobs) as ex:
        for k, recs, rounds, dt in ex.map(run_one, jobs):
            x = data[k][1]["x"]
            out["kernels"][str(k)] = {"count": int(counts[k]), "instr_sum": str(int(x.astype(object).sum())),
                                      "class": int(cls[k]), "rounds": int(rounds), "oracle_s": round(dt, 1)}
            out["strata"] += recs
            print(f"kernel {k}: {counts[k]} invocations, {len(recs)} strata, {rounds} rounds, {dt:.1f} s",
                  flush=True)
    out["strata"].sort(key=lambda r: (r["kernel_id"], r["lo"]))
    with open(OUT, "w") as f:
        json.dump(out, f, indent=0)
    print("wrote", OUT, len(out["strata"]), "strata")


if __name__ == "__main__":
    main()
