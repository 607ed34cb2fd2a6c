"""Per-launch summary of an ncu report: duration, DRAM bytes, throughput, occupancy, IPC.
usage: python tools/ncu_summary.py REPORT [--json OUT]"""
import csv
import io
import json
import subprocess
import sys

rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr, units, data = rows[0], rows[1], rows[2:]
col = {h: i for i, h in enumerate(hdr)}
want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "sm__inst_executed.avg.per_cycle_active",
        "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct", "launch__registers_per_thread",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed"]
res = []
for r in data:
    d = {"id": r[col["ID"]], "kernel": r[col["Kernel Name"]][:60]}
    for w in want:
        if w in col:
            v = r[col[w]].replace(",", "")
            u = units[col[w]]
            try:
                v = float(v)
            except ValueError:
                pass
            # normalise to ns / bytes
            if w == "gpu__time_duration.sum":
                v = v * {"ns": 1, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6, "nsecond": 1}.get(u, 1)
            if w.startswith("dram__bytes"):
                v = v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}.get(u, 1)
            d[w] = v
    res.append(d)
for d in res:
    t = d.get("gpu__time_duration.sum", 0) / 1e3
    rb = d.get("dram__bytes_read.sum", 0) / 1e6
    wb = d.get("dram__bytes_write.sum", 0) / 1e6
    gbs = (rb + wb) / t if t else 0
    print(f"{d['id']:>3} {d['kernel'][:44]:44s} {t:9.1f} us  R {rb:8.1f} MB  W {wb:8.1f} MB  {gbs:7.1f} GB/s  "
          f"occ {d.get('sm__warps_active.avg.pct_of_peak_sustained_active', 0):5.1f}%  ipc {d.get('sm__inst_executed.avg.per_cycle_active', 0):4.2f}  "
          f"L2hit {d.get('lts__t_sector_hit_rate.pct', 0):5.1f}  regs {d.get('launch__registers_per_thread', 0)}")
if len(sys.argv) > 3 and sys.argv[2] == "--json":
    json.dump(res, open(sys.argv[3], "w"), indent=1)
