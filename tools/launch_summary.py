"""Summarise an ncu launch list (--metrics gpu__time_duration.sum[,dram__bytes_read.sum,dram__bytes_write.sum]
--csv): per kernel name, launches, total/mean device time and DRAM bytes, for the last `passes` index
passes (each pass starts with k_warp_kstart).  With --json OUT also writes the per-pass DRAM traffic
(bench.py reads it as roofline.traffic).
usage: python tools/launch_summary.py launches.csv [passes_to_keep] [--json OUT --bmin B]"""
import collections
import csv
import json
import re
import sys

args = [a for a in sys.argv[1:]]
jout = None
bmin = None
if "--json" in args:
    i = args.index("--json")
    jout = args[i + 1]
    del args[i:i + 2]
if "--bmin" in args:
    i = args.index("--bmin")
    bmin = float(args[i + 1])
    del args[i:i + 2]
path = args[0]
keep = int(args[1]) if len(args) > 1 else 1
launch = {}
with open(path) as f:
    lines = [l for l in f if l.startswith('"')]
rd = csv.DictReader(lines)
UNIT = {"nsecond": 1, "usecond": 1e3, "msecond": 1e6, "ns": 1, "us": 1e3, "ms": 1e6}
BUNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}
for r in rd:
    m = r.get("Metric Name")
    v = float(r["Metric Value"].replace(",", ""))
    u = r["Metric Unit"]
    i = int(r["ID"])
    name = re.sub(r"\(.*", "", r["Kernel Name"]).replace("void ", "")
    d = launch.setdefault(i, {"name": name, "ns": 0.0, "dram": 0.0})
    if m == "gpu__time_duration.sum":
        d["ns"] = v * UNIT.get(u, 1)
    elif m in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
        d["dram"] += v * BUNIT.get(u, 1)
rows = [(i, d["name"], d["ns"], d["dram"]) for i, d in sorted(launch.items())]
starts = [k for k, (_, n, _, _) in enumerate(rows) if n.startswith("wj::k_warp_kstart") or n.startswith("k_warp_kstart")]
sel = rows[starts[-keep]:] if len(starts) >= keep else rows
agg = collections.OrderedDict()
for _, n, ns, dr in sel:
    a = agg.setdefault(n, [0, 0.0, 0.0])
    a[0] += 1
    a[1] += ns
    a[2] += dr
tot = sum(a[1] for a in agg.values())
totb = sum(a[2] for a in agg.values())
print(f"{len(sel)} launches, {tot/1e6/keep:.3f} ms per pass (serialised, cold-cache), "
      f"DRAM {totb/1e9/keep:.3f} GB per pass")
for n, (c, ns, dr) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print(f"{100*ns/tot:5.1f}%  {ns/1e6/keep:8.3f} ms/pass  {c/keep:5.1f} launches/pass  {dr/1e9/keep:7.3f} GB/pass  {n}")
if jout:
    per = {n: a[2] / keep for n, a in agg.items()}
    out = {"step_dram_bytes": totb / keep, "per_kernel_dram_bytes": per,
           "_source": f"{path}: dram__bytes_read.sum + dram__bytes_write.sum summed over the launches of one "
                      f"index pass (ncu --clock-control none launch list, cold-cache, serialised)"}
    if bmin:
        out["b_min"] = bmin
        out["traffic_ratio"] = totb / keep / bmin
    json.dump(out, open(jout, "w"), indent=1)
