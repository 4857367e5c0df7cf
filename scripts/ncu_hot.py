"""Hot spots of an ncu report (run here, no GPU): per CUDA source line, the warp-stall samples
and executed warp instructions (report captured with --import-source on, library built with
-lineinfo).  Usage: python scripts/ncu_hot.py REPORT [top] [kernel-regex]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
cmd = ["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"]
if len(sys.argv) > 3:
    cmd += ["--kernel-name", f"regex:{sys.argv[3]}"]
out = subprocess.run(cmd, capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr, fname, lines = None, "", []
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
    elif r[0] == "Line No":
        hdr = r
    elif hdr and r[0].isdigit():
        d = dict(zip(hdr[2:], r[2:]))
        try:
            s = float(d.get("Warp Stall Sampling (All Samples)", "0") or 0)
            i = float(d.get("Instructions Executed", "0") or 0)
        except ValueError:
            continue
        lines.append((s, i, f"{fname}:{r[0]}", r[1].strip()[:70]))
ts = sum(x[0] for x in lines) or 1
ti = sum(x[1] for x in lines) or 1
print(f"total stall samples {ts:.0f}, warp instructions executed {ti:.4e}")
for s, i, where, src in sorted(lines, key=lambda x: -x[0])[:top]:
    print(f"{s / ts * 100:6.2f}% samp {i / ti * 100:6.2f}% inst  {where:28s} {src}")
