"""Summarise an ncu launch list (--metrics gpu__time_duration.sum[,dram__bytes_*] --csv) per kernel:
launches / step, ms / step, DRAM MB / step and GB/s.   python tools/launch_table.py <csv> <steps>"""
import collections
import csv
import sys


def main(path, steps):
    rows = list(csv.reader(open(path)))
    i = [k for k, r in enumerate(rows) if r and r[0] == "ID"][0]
    hdr, data = rows[i], rows[i + 1:]
    ki, mi, vi, ui = (hdr.index(h) for h in ("Kernel Name", "Metric Name", "Metric Value", "Metric Unit"))
    tscale = {"nsecond": 1e-6, "ns": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1.0, "ms": 1.0, "second": 1e3}
    bscale = {"byte": 1e-6, "Kbyte": 1e-3, "Mbyte": 1.0, "Gbyte": 1e3, "B": 1e-6, "KB": 1e-3, "MB": 1.0, "GB": 1e3}
    agg = collections.defaultdict(lambda: collections.defaultdict(float))
    cnt = collections.Counter()
    for r in data:
        name = r[ki].split("(")[0]
        v = float(r[vi].replace(",", ""))
        if r[mi] == "gpu__time_duration.sum":
            cnt[name] += 1
            agg[name]["ms"] += v * tscale[r[ui]]
        else:
            agg[name]["MB"] += v * bscale.get(r[ui], 1e-6)
    tot = sum(a["ms"] for a in agg.values()) / steps
    print(f"{len(data)} rows over {steps} steps; GPU time {tot:.3f} ms/step\n")
    print("| kernel | launches/step | ms/step | share | DRAM MB/step | GB/s |")
    print("|---|---|---|---|---|---|")
    for n, a in sorted(agg.items(), key=lambda x: -x[1]["ms"]):
        ms, mb = a["ms"] / steps, a["MB"] / steps
        print(f"| {n} | {cnt[n] / steps:.1f} | {ms:.4f} | {100 * ms / tot:.1f}% | {mb:.1f} | "
              f"{mb / ms if ms else 0:.0f} |")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]))
