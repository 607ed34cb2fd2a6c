"""One-paragraph summary of a bench.py JSON line (ms/step, roofline, per-kernel and per-phase ms)."""
import json
import sys

d = json.load(open(sys.argv[1]))
print("ms/step", round(d["ms_per_step"], 3), "MB/s", round(d["value"]), "roofline", round(d["roofline"]["frac"], 4),
      "launches", d.get("gpu_launches_per_step"), "syncs", d.get("host_syncs_per_step"))
print("kernels", {k: round(v["ms_per_step"], 3) for k, v in d["kernels"].items() if v["ms_per_step"]})
print("phases", {k: round(v, 3) for k, v in d["phases_ms_per_step"].items() if v})
if d.get("e2e"):
    print("e2e", round(d["e2e"]["value"]), d["e2e"].get("ms_per_step"))
