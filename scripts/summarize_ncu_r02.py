"""Summarise `ncu --set full` captures of the traversal kernel per config (run here, no GPU).

  python scripts/summarize_ncu_r02.py cfg2=gpurun_out/ncu_fill2_cfg2.ncu-rep[:LOG] cfg4=...

LOG (optional) is scripts/prof_count.py's output for the same capture, giving the rows and
vertices scanned (SV) of the profiled pass.  Writes profiles/r02/ncu_summary.json (read by
bench.py's roofline: dram traffic, HBM GB/s, L2 and issue fractions, warp instructions per
scanned vertex) and profiles/r02/ncu_<cfg>.txt (the key metrics, human-readable)."""
import csv
import io
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "profiles", "r02")
KEYS = {"gpu__time_duration.sum": "time", "dram__bytes_read.sum": "dram_read",
        "dram__bytes_write.sum": "dram_write", "lts__t_sectors.sum": "lts_sectors",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed": "l2_pct",
        "sm__issue_active.avg.pct_of_peak_sustained_elapsed": "issue_pct",
        "l1tex__throughput.avg.pct_of_peak_sustained_elapsed": "l1_pct",
        "sm__warps_active.avg.pct_of_peak_sustained_active": "occupancy_pct",
        "smsp__inst_executed.sum": "inst_executed", "launch__grid_size": "grid",
        "launch__block_size": "block", "launch__registers_per_thread": "registers",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum": "smem_bank_conflicts"}
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1, "us": 1e3, "ms": 1e6,
         "s": 1e9}

path = os.path.join(OUT, "ncu_summary.json")
summary = json.load(open(path)) if os.path.exists(path) else {}
for arg in sys.argv[1:]:
    key, spec = arg.split("=", 1)
    cfg, _, kkey = key.partition("/")
    kkey = kkey or "fill2_stage"
    rep, _, log = spec.partition(":")
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    r = list(csv.reader(io.StringIO(raw)))
    hdr, units, row = r[0], r[1], r[2]
    m = {}
    for name, key in KEYS.items():
        if name in hdr:
            k = hdr.index(name)
            v = float(row[k].replace(",", "") or 0)
            m[key] = v * SCALE.get(units[k], 1)
    kname = row[hdr.index("Kernel Name")]
    rec = {"kernel": kname, "time_ns": m["time"], "dram_bytes": m["dram_read"] + m["dram_write"],
           "dram_read": m["dram_read"], "dram_write": m["dram_write"],
           "l2_bytes": m.get("lts_sectors", 0) * 32, "l2_pct": m.get("l2_pct"),
           "issue_pct": m.get("issue_pct"), "l1_pct": m.get("l1_pct"),
           "occupancy_pct": m.get("occupancy_pct"), "inst_executed": m.get("inst_executed"),
           "grid": m.get("grid"), "block": m.get("block"), "registers": m.get("registers"),
           "smem_bank_conflicts": m.get("smem_bank_conflicts"),
           "report": os.path.basename(rep)}
    if log and os.path.exists(log):
        for line in open(log):
            mm = re.search(r"rows \[(\d+),(\d+)\): count ([\d.]+) ms, SV (\d+)", line)
            if mm and "==PROF" not in line:
                rec["rows"] = [int(mm.group(1)), int(mm.group(2))]
                rec["sv"] = int(mm.group(4))
    summary.setdefault(cfg, {})[kkey] = rec
    src = (f"ncu --set full --import-source on of scripts/prof_count.py "
           f"({os.path.basename(rep)}); rows {rec.get('rows', 'all')}")
    if kkey == "fill2_stage":
        summary[cfg]["_source"] = src
    fname = f"ncu_{cfg}.txt" if kkey == "fill2_stage" else f"ncu_{cfg}_{kkey}.txt"
    with open(os.path.join(OUT, fname), "w") as f:
        f.write(f"# {src}\n# kernel: {kname}\n")
        t = rec["time_ns"] / 1e9
        f.write(f"duration_ms            {rec['time_ns'] / 1e6:.3f}\n")
        f.write(f"dram_bytes             {rec['dram_bytes']:.4e}  ({rec['dram_bytes'] / t / 1e9:.1f} GB/s)\n")
        f.write(f"l2_bytes               {rec['l2_bytes']:.4e}  ({rec['l2_bytes'] / t / 1e9:.1f} GB/s)\n")
        for k in ("l2_pct", "issue_pct", "l1_pct", "occupancy_pct", "inst_executed", "grid",
                  "block", "registers", "smem_bank_conflicts", "sv"):
            if rec.get(k) is not None:
                f.write(f"{k:22s} {rec[k]}\n")
        if rec.get("sv"):
            f.write(f"warp_inst_per_sv       {rec['inst_executed'] / rec['sv']:.2f}\n")
json.dump(summary, open(path, "w"), indent=1, sort_keys=True)
print(json.dumps(summary, indent=1)[:3000])
