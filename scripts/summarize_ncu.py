"""Summarise ncu reports (run here, no GPU): python scripts/summarize_ncu.py <round> <cfg>.

Writes profiles/<round>/launches_cfg<cfg>.txt (per-kernel device time and share of the step),
profiles/<round>/ncu_<kernel>_cfg<cfg>.txt (key metrics of the full-set capture) and updates
profiles/traffic.json (DRAM bytes per launch, read by bench.py's roofline.traffic)."""
import csv
import io
import json
import os
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
rnd, cfg = sys.argv[1], sys.argv[2]
out = os.path.join(ROOT, "profiles", rnd)
os.makedirs(out, exist_ok=True)
go = os.path.join(ROOT, "gpurun_out")

# ---- launch list
rows = list(csv.reader(open(os.path.join(go, f"launches_cfg{cfg}.csv"))))
hi = [k for k, r in enumerate(rows) if r and r[0] == "ID"][0]
h = rows[hi]
ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
agg = defaultdict(lambda: [0, 0.0])
for r in rows[hi + 1:]:
    name = r[ki].split("(")[0]
    v = float(r[vi].replace(",", ""))
    v = v / 1e3 if r[ui] == "ns" else (v * 1e3 if r[ui] == "ms" else v)  # -> us
    agg[name][0] += 1
    agg[name][1] += v
tot = sum(x[1] for x in agg.values())
with open(os.path.join(out, f"launches_cfg{cfg}.txt"), "w") as f:
    f.write(f"# ncu --metrics gpu__time_duration.sum --clock-control none, bench.py --profile "
            f"--config {cfg} (warm-up step + 1 step; serialised, cold-cache)\n")
    f.write(f"{'kernel':80s} {'launches':>8s} {'total_us':>12s} {'share':>7s}\n")
    for name, (c, us) in sorted(agg.items(), key=lambda x: -x[1][1]):
        f.write(f"{name[:80]:80s} {c:8d} {us:12.1f} {us / tot * 100:6.2f}%\n")
print(open(os.path.join(out, f"launches_cfg{cfg}.txt")).read())

# ---- full-set captures
WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "lts__t_bytes.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "inst_executed",
        "smsp__inst_executed.avg.per_cycle_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "launch__shared_mem_per_block_dynamic", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct",
        "smsp__pcsamp_warps_issue_stalled_barrier", "smsp__pcsamp_warps_issue_stalled_long_scoreboard",
        "smsp__pcsamp_warps_issue_stalled_short_scoreboard", "smsp__pcsamp_warps_issue_stalled_wait",
        "smsp__pcsamp_warps_issue_stalled_lg_throttle", "smsp__pcsamp_warps_issue_stalled_mio_throttle"]
traffic_path = os.path.join(ROOT, "profiles", "traffic.json")
traffic = json.load(open(traffic_path)) if os.path.exists(traffic_path) else {}
for rep in (f"fill2_cfg{cfg}", f"aux_cfg{cfg}"):
    path = os.path.join(go, rep + ".ncu-rep")
    if not os.path.exists(path):
        continue
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    r = list(csv.reader(io.StringIO(raw)))
    hdr, units = r[0], r[1]
    for row in r[2:]:
        kname = row[hdr.index("Kernel Name")]
        short = kname.split("(")[0].split("::")[-1]
        mode = ""
        if "fill2_kernel" in kname:
            # template args: <NT, W, MODE, VIS>
            args = kname.split("<")[1].split(">")[0].replace("(int)", "").split(",")
            mode = {"0": "count", "1": "emit", "2": "stage"}[args[2].strip()]
            short = f"fill2_{mode}"
        fn = os.path.join(out, f"ncu_{short}_cfg{cfg}.txt")
        with open(fn, "w") as f:
            f.write(f"# ncu --set full --clock-control none: {kname}\n")
            for w in WANT:
                if w in hdr:
                    k = hdr.index(w)
                    f.write(f"{w:70s} {row[k]:>20s} {units[k]}\n")
        k = hdr.index
        def val(m):
            v = row[k(m)].replace(",", "")
            u = units[k(m)]
            x = float(v)
            return x * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
        traffic.setdefault(f"cfg{cfg}", {})[short] = val("dram__bytes_read.sum") + \
            val("dram__bytes_write.sum")
        print(open(fn).read())
json.dump(traffic, open(traffic_path, "w"), indent=1, sort_keys=True)
print(json.dumps(traffic, indent=1))
