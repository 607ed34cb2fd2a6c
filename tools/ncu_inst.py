"""Top CUDA source lines of one kernel in an ncu report by executed warp instructions.
usage: python tools/ncu_inst.py REPORT [N]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                      "--launch-count", "1"], capture_output=True, text=True).stdout
rows, cur, hdr = [], None, None
for line in out.splitlines():
    if line.startswith('"File Path"') or line.startswith('"File Name"'):
        cur = line.split(",", 1)[1].strip('"').split("/")[-1]
        continue
    if line.startswith('"Line No"'):
        hdr = next(csv.reader(io.StringIO(line)))
        continue
    if hdr is None:
        continue
    r = next(csv.reader(io.StringIO(line)))
    if len(r) != len(hdr) or not r[0]:
        continue
    d = dict(zip(hdr, r))
    try:
        inst = int(d.get("Instructions Executed", "0") or 0)
        thr = int(d.get("Thread Instructions Executed", "0") or 0)
    except ValueError:
        continue
    rows.append((inst, thr, cur, d["Line No"], r[1][:100]))
tot = sum(r[0] for r in rows) or 1
print(f"warp instructions {tot}")
for i, t, f, ln, src in sorted(rows, reverse=True)[:n]:
    print(f"{100 * i / tot:5.1f}%  lanes/inst {t / max(i, 1):5.1f}  {f}:{ln}  {src}")
