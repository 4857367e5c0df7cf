"""Warp instructions and stall samples of an ncu source page grouped into line ranges of
fill2_impl.cuh (regions of the traversal).  Usage: python scripts/ncu_regions.py REPORT"""
import csv
import io
import subprocess
import sys

REGIONS = [("block_scan", 65, 92), ("bitmap helpers", 102, 222), ("ell/put/push", 224, 273),
           ("next_word/scan_bits (collect, emit)", 275, 415), ("scan_level (BFS level)", 417, 563),
           ("scan_level_multi", 565, 661), ("bfs loop", 663, 708),
           ("kernel: setup/claim/seed", 710, 833), ("kernel: threshold windows", 834, 960),
           ("kernel: count/stage/emit/clear", 961, 1022)]
out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source",
                      "cuda,sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr, fname, acc = None, "", {}
tot_i = tot_s = 0.0
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
            i = float(d.get("Instructions Executed") or 0)
            s = float(d.get("Warp Stall Sampling (All Samples)") or 0)
        except ValueError:
            continue
        tot_i += i
        tot_s += s
        ln = int(r[0])
        name = fname
        if fname == "fill2_impl.cuh":
            name = next((n for n, a, b in REGIONS if a <= ln <= b), "fill2_impl.cuh other")
        a = acc.setdefault(name, [0.0, 0.0])
        a[0] += i
        a[1] += s
print(f"total warp instructions {tot_i:.4e}, stall samples {tot_s:.0f}")
for k, (i, s) in sorted(acc.items(), key=lambda x: -x[1][0]):
    print(f"  {k:45s} inst {i / tot_i * 100:6.2f}%  samples {s / tot_s * 100:6.2f}%")
