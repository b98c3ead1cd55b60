"""Device-timed measurements of SURVEY 8(f)'s NEXT rows (not the bench contract's line, which is
the a0-a10 path): each call timed with CUDA events on the library's stream after warm-up, median
of the timed repetitions, with the algorithmic bytes of the streaming ones against the measured
HBM copy bandwidth (MEASURED_PEAKS.json).  Prints one JSON object.

    python tools/bench_next.py [--config C4] [--reps 5]

  NEXT-1  stratify_sweep over 10 thetas vs 10 separate stratify calls; tier_census over 10 thetas
  NEXT-2  predict_multi for M = 1 / 8 / 64 architectures; cycle_cov (one pass over sid + cycles)
  NEXT-3  min_strata (exact interval DP over every Tier-3 kernel's distinct values), on C3
  NEXT-4  load_csv of a C3-shaped CSV export from device-resident text and from host text
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def hbm_peak():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        for k in ("hbm_copy_GBps", "hbm_GBps", "copy_GBps"):
            if k in d:
                return float(d[k]), "MEASURED_PEAKS.json " + k
        for k, v in d.items():
            if "hbm" in k.lower() and isinstance(v, (int, float)):
                return float(v), "MEASURED_PEAKS.json " + k
    except (OSError, ValueError):
        pass
    return 6448.1, "fallback"


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C4")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--only", default="", help="comma list of rows to run: next1,next2,next3,next4")
    a = ap.parse_args()
    import numpy as np
    import torch
    import gen
    import paper_conf_ispass_naderantahanse23_b200 as sieve

    stream = torch.cuda.Stream()

    def timed(fn, reps=a.reps, warm=2):
        for _ in range(warm):
            out = fn()
        ts = []
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record(stream)
            out = fn()
            e1.record(stream)
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        return statistics.median(ts), out

    def load(cfg_name):
        cfg = gen.get_config(cfg_name)
        tr = gen.Generator(cfg).fill(0, cfg.n)
        d = {k: torch.from_numpy(tr[k].view(np.int64 if tr[k].dtype == np.uint64 else np.int32)).cuda()
             for k in ("kid", "x", "cta", "y")}
        ctx = sieve.Ctx(device=0, stream=stream)
        t = sieve.load_trace(ctx, d["kid"], d["x"], num_kernels=cfg.K, cta=d["cta"], cycles=d["y"], adopt=True)
        return cfg, tr, d, ctx, t

    only = set(a.only.split(",")) if a.only else {"next1", "next2", "next3", "next4"}
    peak, peak_src = hbm_peak()
    res = {"config": a.config, "hbm_peak_GBps": peak, "hbm_peak_source": peak_src, "reps": a.reps,
           "timing": "CUDA events on the library stream, median of reps after 2 warm-up calls"}
    if only & {"next1", "next2"}:
        next12(a, res, load, timed, sieve, np, torch, peak, only)
    if only & {"next3", "next4"}:
        next34(a, res, load, timed, sieve, np, torch, only)
    print(json.dumps(res))


def next12(a, res, load, timed, sieve, np, torch, peak, only):
    cfg, tr, d, ctx, t = load(a.config)
    ctx.set_term_count(False)
    n = cfg.n
    thetas = [(k, 10) for k in range(1, 11)]

    ms1, _ = timed(lambda: sieve.stratify(t))
    ms_sw, sts = timed(lambda: sieve.stratify_sweep(t, thetas))
    res["stratify_ms"] = ms1
    res["NEXT-1"] = {
        "stratify_sweep_10_thetas_ms": ms_sw,
        "ten_separate_stratify_ms_est": 10 * ms1,
        "sweep_speedup_vs_separate": 10 * ms1 / ms_sw,
        "strata_per_theta": [len(s) for s in sts],
    }
    ms_c, (kk, inv, _) = timed(lambda: sieve.tier_census(t, thetas))
    res["NEXT-1"]["tier_census_10_thetas_ms"] = ms_c
    res["NEXT-1"]["tier_census_invocations_per_s"] = n / (ms_c / 1e3)

    sid = torch.empty(n, dtype=torch.int32, device="cuda")
    st = sieve.stratify(t, stratum_of_invocation=sid)
    ns = len(st)
    rc0 = st.table["rep_cycles"]
    pm = {}
    for M in (1, 8, 64):
        rc = np.stack([rc0 + np.uint64(m) for m in range(M)])
        ms_m, _ = timed(lambda: sieve.predict_multi(st, t, rc))
        pm[f"M={M}_ms"] = ms_m
    ms_p, _ = timed(lambda: sieve.predict(st, t))
    ms_cc, _ = timed(lambda: sieve.cycle_cov(st, t, sid))
    cc_bytes = 12 * n   # sid u32 + cycles u64 per invocation
    res["NEXT-2"] = {"strata": ns, "predict_ms": ms_p, "predict_multi": pm, "cycle_cov_ms": ms_cc,
                     "cycle_cov_alg_bytes": cc_bytes, "cycle_cov_GBps": cc_bytes / (ms_cc / 1e3) / 1e9,
                     "cycle_cov_hbm_frac": cc_bytes / (ms_cc / 1e3) / 1e9 / peak}
    del sid, st, sts, t, d
    torch.cuda.synchronize()


def next34(a, res, load, timed, sieve, np, torch, only):
    cfg3, tr3, d3, ctx3, t3 = load("C3")
    if "next3" in only:   # on C3: the exact DP is O(m^2) per kernel in its distinct values
        ms_dp, (counts, _) = timed(lambda: sieve.min_strata(t3, max_distinct=1 << 20), reps=3, warm=1)
        ok = counts != 0xFFFFFFFF
        st3 = sieve.stratify(t3)
        per = np.bincount(st3.table["kernel_id"], minlength=cfg3.K)
        res["NEXT-3"] = {"config": "C3", "min_strata_ms": ms_dp, "kernels_solved": int(ok.sum()),
                         "optimum_strata": int(counts[ok].sum()), "sieve_strata_same_kernels": int(per[ok].sum())}
    if "next4" not in only:
        return

    # NEXT-4: a C3-shaped CSV export (name, instructions, CTA size, cycles)
    names = np.array([f"void kernel_{k}<float, 128>(float const*, int)" for k in range(cfg3.K)])
    m = 2_000_000
    lines = ["Kernel Name,Instructions,Block Size,Cycles"]
    kid, x, cta, y = tr3["kid"][:m], tr3["x"][:m], tr3["cta"][:m], tr3["y"][:m]
    lines += [f'"{names[k]}",{xi},{ci},{yi}' for k, xi, ci, yi in zip(kid.tolist(), x.tolist(), cta.tolist(), y.tolist())]
    text = ("\n".join(lines) + "\n").encode()
    dev = torch.frombuffer(bytearray(text), dtype=torch.uint8).cuda()
    ms_dev, (tc, nm) = timed(lambda: sieve.load_csv(ctx3, dev, col_kernel=0, col_instr=1, col_cta=2,
                                                      col_cycles=3), reps=3, warm=1)
    ms_host, _ = timed(lambda: sieve.load_csv(ctx3, text, col_kernel=0, col_instr=1, col_cta=2, col_cycles=3),
                       reps=3, warm=1)
    res["NEXT-4"] = {"rows": m, "text_bytes": len(text), "kernels": len(nm),
                     "device_text_ms": ms_dev, "device_text_GBps": len(text) / (ms_dev / 1e3) / 1e9,
                     "device_rows_per_s": m / (ms_dev / 1e3),
                     "host_text_ms": ms_host, "host_text_GBps": len(text) / (ms_host / 1e3) / 1e9}


if __name__ == "__main__":
    main()
