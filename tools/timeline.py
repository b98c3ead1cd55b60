"""GPU timeline of stratify + predict steps (CUPTI through torch.profiler): every kernel's start
and end on the device, the idle gaps between them, and which kernel each gap precedes.

    python tools/timeline.py [--config C4] [--steps 3]
"""
import argparse
import collections
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C4")
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--dump", action="store_true", help="list the last step's kernels and gaps in order")
    a = ap.parse_args()
    import numpy as np
    import torch
    from torch.profiler import ProfilerActivity, profile
    import gen
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    cfg = gen.get_config(a.config)
    tr = gen.Generator(cfg).fill(0, cfg.n)
    d = {k: torch.from_numpy(tr[k].view(np.int64 if tr[k].dtype == np.uint64 else np.int32)).cuda()
         for k in ("kid", "x", "cta", "y")}
    stream = torch.cuda.Stream()
    ctx = sieve.Ctx(device=0, stream=stream)
    t = sieve.load_trace(ctx, d["kid"], d["x"], num_kernels=cfg.K, cta=d["cta"], cycles=d["y"], adopt=True)
    sid = torch.empty(cfg.n, dtype=torch.int32, device="cuda")
    for _ in range(3):
        sieve.predict(sieve.stratify(t, stratum_of_invocation=sid), t)
    ctx.set_term_count(False)
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        for _ in range(a.steps):
            sieve.predict(sieve.stratify(t, stratum_of_invocation=sid), t)
        torch.cuda.synchronize()
    ev = [e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA]
    ev = sorted(ev, key=lambda e: e.time_range.start)
    if not ev:
        print("no CUDA events captured")
        return
    span = ev[-1].time_range.end - ev[0].time_range.start
    busy, gaps, end = 0.0, collections.defaultdict(float), ev[0].time_range.start
    gap_count = collections.Counter()
    for e in ev:
        s, f = e.time_range.start, e.time_range.end
        if s > end:
            g = s - end
            gaps[e.name.split("(")[0][:40]] += g
            gap_count[e.name.split("(")[0][:40]] += 1
            busy += f - s
            end = f
        else:
            busy += max(0.0, f - end)
            end = max(end, f)
    per = a.steps
    # the largest single gaps with their neighbours (one step's worth)
    singles = []
    for p_, e in zip(ev[:-1], ev[1:]):
        g = e.time_range.start - p_.time_range.end
        if g > 0:
            singles.append((g, p_.name.split("(")[0][:32], e.name.split("(")[0][:32]))
    singles.sort(reverse=True)
    print("largest gaps (us): " + "; ".join(f"{g:.1f} {a_} -> {b_}" for g, a_, b_ in singles[:3 * per + 6]))
    print(f"{len(ev)} device events over {per} steps: span {span / 1e3 / per:.3f} ms/step, busy "
          f"{busy / 1e3 / per:.3f} ms/step, idle {(span - busy) / 1e3 / per:.3f} ms/step "
          f"(between the first and the last kernel)")
    if a.dump:   # the last step: every device event with its start (us from the step's first) and the gap
        starts = [i for i, e in enumerate(ev) if e.name.startswith("k_moments") and "reduce" not in e.name]
        first = starts[-1] if starts else 0
        t0 = ev[first].time_range.start
        prev_end = ev[first - 1].time_range.end if first else t0
        for e in ev[first:]:
            s_, f_ = e.time_range.start, e.time_range.end
            print(f"{(s_ - t0):9.1f} {(f_ - s_):8.1f} gap {max(0.0, s_ - prev_end):6.1f}  {e.name.split('(')[0][:48]}")
            prev_end = max(prev_end, f_)
    print("| idle before kernel | us/step | gaps/step |\n|---|---|---|")
    for k, v in sorted(gaps.items(), key=lambda x: -x[1])[:25]:
        print(f"| {k} | {v / per:.1f} | {gap_count[k] / per:.1f} |")


if __name__ == "__main__":
    main()
