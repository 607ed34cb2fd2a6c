"""Per CUDA source line: instructions executed and stall samples from an ncu report
(--page source --print-source cuda,sass).  usage: python tools/ncu_lines_cuda.py REPORT [top]"""
import csv
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows, f, hdr = [], None, None
for r in csv.reader(out.splitlines()):
    if len(r) == 2 and r[0] == "File Path":
        f = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if hdr and len(r) == len(hdr) and r[0] not in ("-", ""):
        rows.append((f, r[0], r[1], int(r[7] or 0) if r[7] not in ("-",) else 0, int(r[4]) if r[4] not in ("-", "") else 0))
ti = sum(x[3] for x in rows)
ts = sum(x[4] for x in rows)
print(f"total warp-instructions {ti}, stall samples {ts}")
for f, ln, src, ins, smp in sorted(rows, key=lambda x: -x[4])[:top]:
    print(f"{f[:14]:14s} {ln:>5s} inst {ins / max(ti, 1) * 100:5.1f}% stall {smp / max(ts, 1) * 100:5.1f}%  {src.strip()[:90]}")
