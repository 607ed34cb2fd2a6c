"""Top CUDA source lines of one kernel in an ncu report, by warp-stall samples and instructions.
usage: python tools/ncu_lines.py REPORT LAUNCH_INDEX [N]"""
import csv
import io
import subprocess
import sys

rep, idx = sys.argv[1], int(sys.argv[2])
n = int(sys.argv[3]) if len(sys.argv) > 3 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                      "--launch-skip", str(idx), "--launch-count", "1"], capture_output=True, text=True).stdout
rows, cur_file, hdr = [], None, None
for line in out.splitlines():
    if line.startswith('"File Path"') or line.startswith('"File Name"'):
        cur_file = line.split(",", 1)[1].strip('"').split("/")[-1]
        continue
    if line.startswith('"Function Name"'):
        continue
    if line.startswith('"Line No"'):
        hdr = next(csv.reader(io.StringIO(line)))
        continue
    if hdr is None:
        continue
    r = next(csv.reader(io.StringIO(line)))
    if len(r) != len(hdr):
        continue
    if not r[0]:
        continue  # SASS row
    d = dict(zip(hdr, r))
    d["Source"] = r[1]
    try:
        stall = int(d.get("Warp Stall Sampling (All Samples)", "0") or 0)
        inst = int(d.get("Instructions Executed", "0") or 0)
    except ValueError:
        continue
    rows.append((stall, inst, cur_file, d["Line No"], d["Source"][:110]))
tot_s = sum(r[0] for r in rows) or 1
tot_i = sum(r[1] for r in rows) or 1
print(f"total stall samples {tot_s}, warp instructions {tot_i}")
for s, i, f, ln, src in sorted(rows, reverse=True)[:n]:
    print(f"{100*s/tot_s:5.1f}% st {100*i/tot_i:5.1f}% in  {f}:{ln}  {src}")
