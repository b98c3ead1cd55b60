"""Print the headline numbers of a bench.py JSON log (last JSON line)."""
import json
import sys

for line in open(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/bench.log"):
    line = line.strip()
    if not line.startswith("{"):
        continue
    d = json.loads(line)
    ph = {k: round(v["ms_per_step"], 3) for k, v in d.get("phases", {}).items()}
    roof = d.get("roofline", {})
    print(f"value {d['value']:.4g} ms/step {d['ms_per_step']:.3f} kde frac {roof.get('frac', 0):.3f} "
          f"e2e {(d.get('e2e') or {}).get('value', 0):.3g} clocks {d.get('clocks')}")
    print("phases", ph)
    print("host", d.get("host_ms_per_step"), "launches", d.get("gpu_launches"),
          "eval/inwin", roof.get("evaluated_per_in_window"))
