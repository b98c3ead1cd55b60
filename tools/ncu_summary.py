"""Summarise ncu evidence for profiles/ (run here, on the CPU box, over reports from gpurun_out/).

    python tools/ncu_summary.py launches gpurun_out/launches_r01.csv --steps 5 > profiles/r01_launches.md
    python tools/ncu_summary.py report gpurun_out/prof_kde_r01.ncu-rep > profiles/r01_kde_ncu.md
    python tools/ncu_summary.py traffic gpurun_out/prof_kde_r01.ncu-rep k_kde > profiles/kde_traffic.json
"""
import collections
import csv
import io
import json
import subprocess
import sys

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "dram read"),
    ("dram__bytes_write.sum", "dram write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram % peak"),
    ("sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active", "fp64 pipe %"),
    ("sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active", "alu pipe %"),
    ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "lsu pipe %"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active %"),
    ("launch__registers_per_thread", "regs"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio", "stall long_sb"),
    ("smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio", "stall math"),
    ("smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio", "stall not_sel"),
    ("smsp__average_warps_issue_stalled_wait_per_issue_active.ratio", "stall wait"),
    ("smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio", "stall barrier"),
    ("smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio", "stall mio"),
    ("smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio", "stall short_sb"),
]

TO_BYTES = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
TO_MS = {"nsecond": 1e-6, "usecond": 1e-3, "msecond": 1.0, "us": 1e-3, "ms": 1.0, "ns": 1e-6}


def raw_rows(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True,
                         check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    return [(dict(zip(hdr, r)), dict(zip(hdr, units))) for r in rows[2:] if len(r) == len(hdr)]


def fmt(v, unit):
    return f"{v} {unit}".strip()


def report(rep):
    print(f"# ncu --set full summary: `{rep}`\n")
    print("| kernel | " + " | ".join(n for _, n in KEYS) + " |")
    print("|---|" + "---|" * len(KEYS))
    for r, u in raw_rows(rep):
        name = r.get("Kernel Name", "?").split("(")[0]
        print(f"| {name} | " + " | ".join(fmt(r.get(k, ""), u.get(k, "")) for k, _ in KEYS) + " |")


def traffic(rep, kname):
    per = []
    for r, u in raw_rows(rep):
        base = r.get("Kernel Name", "").split("(")[0]
        base = base[5:] if base.startswith("void ") else base
        if base.split("<")[0] != kname:
            continue
        b = 0.0
        for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            b += float(r[k].replace(",", "")) * TO_BYTES[u[k]]
        per.append(b)
    print(json.dumps({"kernel": kname, "source": rep, "launches": len(per),
                      "dram_bytes_per_launch": sum(per) / max(1, len(per)),
                      "dram_bytes_each": per}))


def launches(path, steps):
    rows = list(csv.reader(open(path)))
    hdr = None
    tot = collections.defaultdict(float)
    cnt = collections.Counter()
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if not hdr or len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        if d["Metric Name"] != "gpu__time_duration.sum":
            continue
        name = d["Kernel Name"].split("(")[0]
        tot[name] += float(d["Metric Value"].replace(",", "")) * TO_MS[d["Metric Unit"]]
        cnt[name] += 1
    S = sum(tot.values())
    print(f"# ncu launch list `{path}` (gpu__time_duration.sum, --clock-control none; cold-cache, "
          f"serialised: compare SHARES)\n")
    print(f"{sum(cnt.values())} launches over {steps} steps; GPU time {S / steps:.3f} ms/step\n")
    print("| kernel | launches/step | ms/step | share |")
    print("|---|---|---|---|")
    for k, v in sorted(tot.items(), key=lambda x: -x[1]):
        print(f"| {k} | {cnt[k] / steps:g} | {v / steps:.4f} | {100 * v / S:.1f}% |")


if __name__ == "__main__":
    mode = sys.argv[1]
    if mode == "report":
        report(sys.argv[2])
    elif mode == "traffic":
        traffic(sys.argv[2], sys.argv[3])
    elif mode == "launches":
        steps = int(sys.argv[sys.argv.index("--steps") + 1]) if "--steps" in sys.argv else 1
        launches(sys.argv[2], steps)
