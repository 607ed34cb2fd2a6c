"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv): per kernel name, launches
and total/mean device time, for the last `--steps` index passes (each pass starts with k_warp_kstart).
usage: python tools/launch_summary.py launches.csv [passes_to_keep]"""
import collections
import csv
import re
import sys

path = sys.argv[1]
keep = int(sys.argv[2]) if len(sys.argv) > 2 else 1
rows = []
with open(path) as f:
    lines = [l for l in f if l.startswith('"')]
rd = csv.DictReader(lines)
for r in rd:
    if r.get("Metric Name") != "gpu__time_duration.sum":
        continue
    v = float(r["Metric Value"].replace(",", ""))
    u = r["Metric Unit"]
    ns = v * {"nsecond": 1, "usecond": 1e3, "msecond": 1e6, "ns": 1, "us": 1e3, "ms": 1e6}.get(u, 1)
    name = re.sub(r"\(.*", "", r["Kernel Name"]).replace("void ", "")
    rows.append((int(r["ID"]), name, ns))
rows.sort()
starts = [i for i, (_, n, _) in enumerate(rows) if n.startswith("wj::k_warp_kstart") or n.startswith("k_warp_kstart")]
sel = rows[starts[-keep]:] if len(starts) >= keep else rows
agg = collections.OrderedDict()
for _, n, ns in sel:
    a = agg.setdefault(n, [0, 0.0])
    a[0] += 1
    a[1] += ns
tot = sum(a[1] for a in agg.values())
print(f"{len(sel)} launches, {tot/1e6/keep:.3f} ms per pass (serialised, cold-cache)")
for n, (c, ns) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print(f"{100*ns/tot:5.1f}%  {ns/1e6/keep:8.3f} ms/pass  {c/keep:5.1f} launches/pass  {n}")
